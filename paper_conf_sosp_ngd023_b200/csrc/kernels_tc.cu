// K2a: convolution as implicit GEMM on the 5th-generation tensor cores (sm_100a).
//
//   D[Cout x P] = W[Cout x K] . im2col(X)[K x P],   K = kh*kw*cin ordered (r, s, ci)
//
// Batch-1 CNN layers have small P (HW down to 49) and Cout >= 64, so the GEMM is
// "swap-AB": Cout is the 128-row UMMA M (= TMEM lanes), output pixels are N = 64.
//
//  * A (weights, [Cout_pad][Kpad] bf16, K-major) is fed by TMA: a 2D tiled tensor
//    map, box 64 (k) x 128 (rows), 128-byte swizzle -- exactly the UMMA K-major
//    SWIZZLE_128B canonical layout;
//  * B (the im2col gather of NHWC activations, with padding, stride, channel stride
//    and channel offset of concat buffers) is gathered by 4 producer warps with
//    16-byte cp.async (zero-fill for padding) into the same swizzled layout;
//  * one elected thread of the MMA warp issues tcgen05.mma.cta_group::1.kind::f16
//    (bf16 x bf16 -> fp32 in TMEM), 4 x K=16 per 64-wide k-block, and releases each
//    smem stage with tcgen05.commit -> mbarrier (4-stage ring);
//  * epilogue: the 4 producer warps read the accumulator with tcgen05.ld (warp w
//    owns TMEM lanes 32w..32w+31 = 32 output channels), add bias, residual (fp32),
//    activation, round once to bf16 (reading C1-Q7) and store NHWC;
//  * split-K over blockIdx.z for the deep, narrow late layers: the ksplit CTAs of a
//    tile form a thread-block cluster; each adds its partial tile into an fp32 workspace
//    with one bulk L2 reduction, and after a cluster barrier each CTA finishes a
//    1/ksplit slice of the tile from the sums (LF_SPLIT_DSMEM: the previous reduction
//    over DSMEM, kept for A/B measurements).
//
// Block instrumentation (K1) wraps the whole CTA (instr.cuh).
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include "common.h"
#include "instr.cuh"
#include "kernels.h"

namespace paella {

namespace {

constexpr uint32_t A_BYTES = TC_BM * TC_BK * 2;   // 16 KiB
constexpr uint32_t B_BYTES = TC_BN * TC_BK * 2;   // 8 KiB
constexpr uint32_t NPROD = 128;                   // producer threads (warps 0-3)

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(b)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n}" ::"r"(su32(b)),
      "r"(parity)
      : "memory");
}
// non-suspending poll (A/B against try_wait's potentially-suspending wait)
__device__ __forceinline__ void mbar_wait_spin(uint64_t* b, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "SPIN_%=:\n\t"
      "mbarrier.test_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra SPIN_%=;\n}" ::"r"(su32(b)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, uint64_t* bar, int x, int y) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
          su32(dst)),
      "l"(map), "r"(su32(bar)), "r"(x), "r"(y)
      : "memory");
}
// B tile by TMA im2col: BN output pixels from linear pixel (w, h) onwards (traversal in
// W, H order with the map's conv strides), 64 channels from c of filter tap (s, r)
__device__ __forceinline__ void tma_im2col_4d(void* dst, const void* map, uint64_t* bar, int c, int w, int h,
                                              uint16_t s, uint16_t r) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.im2col.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4, %5, %6}], [%2], {%7, %8};" ::"r"(su32(dst)),
      "l"(map), "r"(su32(bar)), "r"(c), "r"(w), "r"(h), "r"(0), "h"(s), "h"(r)
      : "memory");
}
__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src, uint32_t src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(src_bytes) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async_global() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// UMMA shared-memory descriptor, K-major, SWIZZLE_128B: 8-row x 128-byte atoms,
// stride between 8-row groups (SBO) 1024 B; version 1 (sm_100); layout type 2.
__device__ __forceinline__ uint64_t sdesc_sw128(uint32_t saddr) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr & 0x3FFFF) >> 4);        // start address
  d |= (uint64_t)(16 >> 4) << 16;                  // LBO (unused for SW128 K-major)
  d |= (uint64_t)(1024 >> 4) << 32;                // SBO
  d |= (uint64_t)1 << 46;                          // descriptor version (sm_100)
  d |= (uint64_t)2 << 61;                          // SWIZZLE_128B
  return d;
}

// instruction descriptor, kind::f16: D=F32, A=B=BF16, both K-major, N, M
__host__ __device__ constexpr uint32_t idesc_bf16(uint32_t M, uint32_t N) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((N >> 3) << 17) | ((M >> 4) << 24);
}

__device__ __forceinline__ void umma_bf16(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                          uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void umma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(bar))
               : "memory");
}

// 32 lanes x 32 bit, 16 consecutive columns per thread
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, float (&v)[16]) {
  uint32_t r[16];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
}

__device__ __forceinline__ float act_tc(float x, uint32_t act) {
  if (act == 1) return fmaxf(x, 0.f);
  if (act == 2) return fminf(fmaxf(x, 0.f), 6.f);
  return x;
}

}  // namespace

// epilogue of one (pixel, 8-channel group) item: bias, residual (fp32), activation,
// one RNE rounding, one 16-byte store
__device__ __forceinline__ void epi_store8(const LayerArgs& a, uint32_t p, uint32_t co, const float (&v)[8],
                                           const float (&bias)[8], const uint4& res) {
  float x[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) x[i] = v[i] + bias[i];
  if (a.flags & LF_RESIDUAL) {
    const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&res);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      float2 f = __bfloat1622float2(h[i]);
      x[2 * i] += f.x;
      x[2 * i + 1] += f.y;
    }
  }
  uint4 o;
  __nv_bfloat162* oh = reinterpret_cast<__nv_bfloat162*>(&o);
#pragma unroll
  for (int i = 0; i < 4; ++i) oh[i] = __floats2bfloat162_rn(act_tc(x[2 * i], a.act), act_tc(x[2 * i + 1], a.act));
  *reinterpret_cast<uint4*>(static_cast<__nv_bfloat16*>(a.out) + (size_t)p * a.out_cs + a.out_co + co) = o;
}

__device__ __forceinline__ void load_bias8(const LayerArgs& a, uint32_t co, float (&b)[8]) {
  if (co < a.cout) {
    const float4 b0 = __ldg(reinterpret_cast<const float4*>(a.bias + co));
    const float4 b1 = __ldg(reinterpret_cast<const float4*>(a.bias + co + 4));
    b[0] = b0.x; b[1] = b0.y; b[2] = b0.z; b[3] = b0.w;
    b[4] = b1.x; b[5] = b1.y; b[6] = b1.z; b[7] = b1.w;
  }
}

__device__ __forceinline__ uint4 load_res8(const LayerArgs& a, uint32_t p, uint32_t co) {
  return __ldg(reinterpret_cast<const uint4*>(static_cast<const __nv_bfloat16*>(a.res) + (size_t)p * a.res_cs +
                                              a.res_co + co));
}

// ksplit == 1 epilogue of one thread: 8 items (pixel px0 + 8 i, channel group g),
// activation and residual fixed at compile time so the unrolled items carry no
// branches and interleave (a single warp per SM sub-partition runs this: its speed
// is instruction latency, not bandwidth); one output pointer advanced by 8 pixels.
template <uint32_t ACT, bool RES, uint32_t NIT, uint32_t BM>
__device__ __forceinline__ void epi_tile(const LayerArgs& a, const float* stage, uint32_t n0, uint32_t P,
                                         uint32_t g, uint32_t co, const float (&bias)[8],
                                         const uint4 (&res)[NIT]) {
  const uint32_t px0 = threadIdx.x / (BM / 8);
  __nv_bfloat16* out = static_cast<__nv_bfloat16*>(a.out) + (size_t)(n0 + px0) * a.out_cs + a.out_co + co;
  const size_t ostep = (size_t)(NPROD / (BM / 8)) * a.out_cs;
  // all items are computed (the staged tile has 64 pixel rows), only the stores are
  // predicated: no branches around the item bodies, so the compiler interleaves them
#pragma unroll
  for (uint32_t i = 0; i < NIT; ++i) {
    const uint32_t px = px0 + i * (NPROD / (BM / 8));
    const float4* q = reinterpret_cast<const float4*>(stage + px * BM + g * 8);
    const float4 u0 = q[0], u1 = q[1];
    float x[8] = {u0.x + bias[0], u0.y + bias[1], u0.z + bias[2], u0.w + bias[3],
                  u1.x + bias[4], u1.y + bias[5], u1.z + bias[6], u1.w + bias[7]};
    if constexpr (RES) {
      const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&res[i]);
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const float2 f = __bfloat1622float2(h[j]);
        x[2 * j] += f.x;
        x[2 * j + 1] += f.y;
      }
    }
    uint4 o;
    __nv_bfloat162* oh = reinterpret_cast<__nv_bfloat162*>(&o);
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      float y0 = x[2 * j], y1 = x[2 * j + 1];
      if constexpr (ACT >= 1) { y0 = fmaxf(y0, 0.f); y1 = fmaxf(y1, 0.f); }
      if constexpr (ACT == 2) { y0 = fminf(y0, 6.f); y1 = fminf(y1, 6.f); }
      oh[j] = __floats2bfloat162_rn(y0, y1);
    }
    if (n0 + px < P) *reinterpret_cast<uint4*>(out) = o;
    out += ostep;
  }
}

// 2 CTAs per SM (two jobs' convs can share an SM): <= 168 registers.  Warp 5 does
// only the block bookkeeping (instrumentation), so no compute warp waits on its
// atomics at entry.
constexpr uint32_t TBOOK = NPROD + 32;   // warp 5, lane 0
template <bool INSTR, bool PRO, uint32_t BN, uint32_t BM = TC_BM>
__global__ void __launch_bounds__(TC_THREADS, 2)
    k_conv_tc(const __grid_constant__ LayerArgs a, const __grid_constant__ InstrArgs ia,
              const __grid_constant__ CUtensorMap wmap) {
  const bool trace = (a.flags & LF_TRACE) != 0;
  const bool spin = (a.flags & LF_MBAR_SPIN) != 0;
  const bool tmab = !PRO && (a.flags & LF_TMA_B) && a.bmap != nullptr;
  uint64_t* tr = trace ? a.trace +
                             16 * ((blockIdx.z * gridDim.y + blockIdx.y) * gridDim.x + blockIdx.x)
                       : nullptr;
  if (trace && threadIdx.x == 0) tr[0] = globaltimer();
  instr_enter<INSTR, TBOOK>(ia);
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // 1024-byte aligned (SW128 atoms); pointer arithmetic on smem_raw (not an integer
  // cast) keeps the shared address space visible to the compiler: LDS/STS, no
  // aliasing with global stores
  uint8_t* smem = smem_raw + ((1024u - (su32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sA = smem;                                  // STAGES x 16 KiB
  constexpr uint32_t BNB = BN * TC_BK * 2;                      // B stage bytes: 8 / 16 KiB
  constexpr uint32_t ABY = BM * TC_BK * 2;                      // A stage bytes: 16 / 8 KiB (M 128 / 64)
  constexpr uint32_t NST = TC_RING / (ABY + BNB);           // 4 stages (BN 64) / 3 (BN 128) / 6 (M 64)
  static_assert(NST <= 16, "barrier arrays hold 16 stages");
  constexpr uint32_t RPT = BN / 16;                             // B pixel rows per gather thread
  uint8_t* sB = smem + NST * ABY;
  uint64_t* full = (uint64_t*)(smem + TC_RING);
  uint64_t* empty = full + 16;
  uint64_t* accb = empty + 16;
  uint64_t* rbar = accb + 1;                           // split-K: peers' slices landed
  uint32_t* tmem_slot = (uint32_t*)(rbar + 1);
  float* stage = reinterpret_cast<float*>(smem);       // epilogue tile [64 px][128 ch] fp32 (reuses sA)

  const uint32_t warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const uint32_t tile_n = blockIdx.x, tile_m = blockIdx.y, split = blockIdx.z;
  const uint32_t P = a.oh * a.ow;
  const uint32_t n0 = tile_n * BN, m0 = tile_m * BM;
  const uint32_t nk = a.kpad / TC_BK;
  const uint32_t per = (nk + a.ksplit - 1) / a.ksplit;
  const uint32_t kb0 = split * per;
  const uint32_t kb1 = min(nk, kb0 + per);
  const uint32_t nkl = kb1 > kb0 ? kb1 - kb0 : 0;

  const uint32_t pre = nkl < NST ? nkl : NST;
  // narrow layers (Cout < 128) fetch only a_rows weight rows per stage; rows a_rows..127
  // of every A stage are zeroed once below (the UMMA still runs M = 128)
  const uint32_t abytes = a.a_rows * 128;
  // LF_TMA_B: k-block kb is filter tap (r, s) = divmod(kb * 64 / cin, kw), channels
  // kb * 64 % cin onwards; the tile's first output pixel's window starts at (tw0, th0)
  const int tw0 = (int)((n0 % a.ow) * a.sw) - (int)a.pw, th0 = (int)((n0 / a.ow) * a.sh) - (int)a.ph;
  auto tma_B = [&](uint32_t it) {
    const uint32_t k0 = (kb0 + it) * TC_BK, tap = k0 / a.cin, c0 = k0 - tap * a.cin;
    const uint32_t r = tap / a.kw, sx = tap - r * a.kw;
    tma_im2col_4d(sB + (it % NST) * BNB, a.bmap, &full[it % NST], (int)c0, tw0, th0, (uint16_t)sx, (uint16_t)r);
  };
  if (warp == 4 && lane == 0) {
    // the MMA warp's leader sets up the barriers and starts the weight stream while
    // the gather warps compute their addresses
    for (uint32_t s = 0; s < NST; ++s) {
      mbar_init(&full[s], tmab ? 1 : NPROD + 1);
      mbar_init(&empty[s], 1);
    }
    mbar_init(accb, 1);
    mbar_init(rbar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    if (trace) tr[11] = globaltimer();
    for (uint32_t it = 0; it < pre; ++it) {   // the first stages need no empty-wait
      mbar_arrive_tx(&full[it], abytes + (tmab ? BNB : 0u));
      tma_load_2d(sA + it * ABY, &wmap, &full[it], (int)((kb0 + it) * TC_BK), (int)m0);
    }
    if (tmab) {   // the activations once the predecessor's output is complete (PDL)
      pdl_wait();
      for (uint32_t it = 0; it < pre; ++it) tma_B(it);
    }
    if (trace) tr[12] = globaltimer();
  }
  // epilogue operands that do not depend on the accumulator: the bias (a weight) is
  // fetched before the PDL wait, the residual right after it, both hidden behind the
  // main loop.  Thread t owns channel group eg = t % 16 and pixels t / 16 + 8 i.
  const uint32_t eg = threadIdx.x % (BM / 8), eco = m0 + eg * 8;
  constexpr uint32_t NIT = BN * (BM / 8) / NPROD;   // 8 items per thread (BN 64)
  float ebias[8];
  uint4 eres[NIT];
  if (warp < 4 && a.ksplit == 1) load_bias8(a, eco, ebias);
  // ---- producer state (warps 0-3): this thread gathers 16-byte chunk `chunk` of
  // pixel rows n = t/8 + 16 j (j < RPT) of every B stage
  const __nv_bfloat16* X = static_cast<const __nv_bfloat16*>(a.in);
  const uint32_t t = threadIdx.x;
  const uint32_t chunk = t % 8;
  // per pixel row j: top-left input coordinate of its window (invalid pixels get a
  // coordinate that fails every bounds check) and its element offset; per stage only
  // the (r, s, ci) offset `dk`, common to the 4 rows, changes
  int ih0[RPT], iw0[RPT], off0[RPT];
  const uint32_t K = a.kh * a.kw * a.cin;
  const uint32_t dst0 = (t / 8) * 128 + ((chunk ^ ((t / 8) & 7)) << 4);   // row t/8 of the SW128 atom
  // (r, s, ci) of k = kbase + 8*chunk, advanced incrementally by TC_BK per stage
  int kr = 0, ks_ = 0, kci = 0;
  uint32_t kcur = 0;
  auto issue_B = [&](uint32_t it, bool arrive) {
    const uint32_t s = it % NST;
    const bool kv = kcur < K;
    const int dk = (kr * (int)a.w_ + ks_) * (int)a.in_cs + kci;
    const uint32_t bstage = su32(sB + s * BNB) + dst0;
#pragma unroll
    for (uint32_t j = 0; j < RPT; ++j) {
      const bool ok = kv && (uint32_t)(ih0[j] + kr) < a.h && (uint32_t)(iw0[j] + ks_) < a.w_;
      const __nv_bfloat16* src = ok ? X + (off0[j] + dk) : X;
      const uint32_t dst = bstage + j * 2048;   // pixel row n = t/8 + 16 j
      cp_async16(dst, src, ok ? 16u : 0u);
    }
    if constexpr (PRO) {
      // DenseNet pre-activation: the raw tile lands by cp.async like the plain path;
      // transform_B applies relu(scale * x + shift) in place once it has landed.  Warm
      // L1 with this chunk's prologue vectors meanwhile.
      if (kv) {
        asm volatile("prefetch.global.L1 [%0];" ::"l"(a.pro_scale + kci));
        asm volatile("prefetch.global.L1 [%0];" ::"l"(a.pro_shift + kci));
      }
    }
    if constexpr (!PRO) {
      // the stage's full barrier is arrived on by the hardware once this thread's
      // copies have landed: the gather warps never wait for their own loads
      if (arrive)
        asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(su32(&full[s])) : "memory");
    }
    // advance (r, s, ci) by TC_BK channels for the next stage
    kcur += TC_BK;
    kci += TC_BK;
    while (kci >= (int)a.cin) {
      kci -= (int)a.cin;
      if (++ks_ == (int)a.kw) {
        ks_ = 0;
        ++kr;
      }
    }
  };
  // PRO: the transform cursor (r, s, ci, k) trails the issue cursor by the stages in flight
  int tr_r = 0, tr_s = 0, tr_ci = 0;
  uint32_t tr_k = 0;
  auto transform_B = [&](uint32_t it) {
    const uint32_t bstage = su32(sB + (it % NST) * BNB) + dst0;
    if (tr_k < K) {
      const float4 s0 = __ldg(reinterpret_cast<const float4*>(a.pro_scale + tr_ci));
      const float4 s1 = __ldg(reinterpret_cast<const float4*>(a.pro_scale + tr_ci + 4));
      const float4 z0 = __ldg(reinterpret_cast<const float4*>(a.pro_shift + tr_ci));
      const float4 z1 = __ldg(reinterpret_cast<const float4*>(a.pro_shift + tr_ci + 4));
      const float sc[8] = {s0.x, s0.y, s0.z, s0.w, s1.x, s1.y, s1.z, s1.w};
      const float sh[8] = {z0.x, z0.y, z0.z, z0.w, z1.x, z1.y, z1.z, z1.w};
#pragma unroll
      for (uint32_t j = 0; j < RPT; ++j) {
        // padding and empty pixels stay zero (padding pads the activated tensor)
        if ((uint32_t)(ih0[j] + tr_r) < a.h && (uint32_t)(iw0[j] + tr_s) < a.w_) {
          const uint32_t adr = bstage + j * 2048;
          uint4 u;
          asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
                       : "=r"(u.x), "=r"(u.y), "=r"(u.z), "=r"(u.w)
                       : "r"(adr));
          __nv_bfloat162* h = reinterpret_cast<__nv_bfloat162*>(&u);
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const float2 f = __bfloat1622float2(h[i]);
            h[i] = __floats2bfloat162_rn(fmaxf(fmaf(sc[2 * i], f.x, sh[2 * i]), 0.f),
                                         fmaxf(fmaf(sc[2 * i + 1], f.y, sh[2 * i + 1]), 0.f));
          }
          asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(adr), "r"(u.x), "r"(u.y), "r"(u.z),
                       "r"(u.w)
                       : "memory");
        }
      }
    }
    tr_k += TC_BK;
    tr_ci += TC_BK;
    while (tr_ci >= (int)a.cin) {
      tr_ci -= (int)a.cin;
      if (++tr_s == (int)a.kw) {
        tr_s = 0;
        ++tr_r;
      }
    }
  };
  if (warp < 4) {
#pragma unroll
    for (uint32_t j = 0; j < RPT; ++j) {
      const uint32_t p = n0 + t / 8 + 16 * j;
      const bool pv = p < P;
      const int oh = (int)(p / a.ow), ow = (int)(p - (uint32_t)oh * a.ow);
      ih0[j] = pv ? oh * (int)a.sh - (int)a.ph : -(1 << 20);
      iw0[j] = pv ? ow * (int)a.sw - (int)a.pw : -(1 << 20);
      off0[j] = pv ? (ih0[j] * (int)a.w_ + iw0[j]) * (int)a.in_cs + (int)a.in_co : 0;
    }
    {
      const uint32_t k0 = kb0 * TC_BK + chunk * 8;
      kcur = k0;
      kci = (int)(k0 % a.cin);
      const int rs = (int)(k0 / a.cin);
      ks_ = rs % (int)a.kw;
      kr = rs / (int)a.kw;
      tr_k = kcur, tr_ci = kci, tr_s = ks_, tr_r = kr;
    }
    if (a.a_rows < BM) {
      const uint32_t zb = ABY - abytes;   // bytes per stage, multiple of 1024
      for (uint32_t o = t * 16; o < NST * zb; o += NPROD * 16) {
        const uint32_t st = o / zb;
        asm volatile("st.shared.v4.u32 [%0], {%1, %1, %1, %1};" ::"r"(su32(sA + st * ABY + abytes + (o - st * zb))),
                     "r"(0u)
                     : "memory");
      }
      fence_proxy_async();   // visible to the tensor core (async proxy) after the CTA barrier
    }
    // ... and the first activation gathers, before the CTA-wide barrier, once the
    // predecessor kernel's output is complete (PDL; the weight TMA above needs no wait)
    pdl_wait();
    if (!tmab)
      for (uint32_t it = 0; it < pre; ++it) {   // barriers not initialised yet
        issue_B(it, false);
        if constexpr (PRO) cp_async_commit();   // one group per stage
      }
    if (a.ksplit == 1 && (a.flags & LF_RESIDUAL) && eco < a.cout) {
#pragma unroll
      for (uint32_t i = 0; i < NIT; ++i) {
        const uint32_t p = n0 + t / (BM / 8) + i * (NPROD / (BM / 8));
        if (p < P) eres[i] = load_res8(a, p, eco);
      }
    }
    if (trace && t == 0) tr[13] = globaltimer();
  }
  __syncthreads();
  if (trace && threadIdx.x == 0) tr[1] = globaltimer();

  if (warp < 4) {
    // ------------------------------------------------------------ producers
    if constexpr (!PRO) {
      if (tmab) {
        // one thread streams both operands by TMA (A + B bytes on one full barrier)
        if (t == 0)
          for (uint32_t nxt = NST; nxt < nkl; ++nxt) {
            const uint32_t s = nxt % NST;
            mbar_wait(&empty[s], ((nxt / NST) & 1) ^ 1);
            mbar_arrive_tx(&full[s], abytes + BNB);
            tma_load_2d(sA + s * ABY, &wmap, &full[s], (int)((kb0 + nxt) * TC_BK), (int)m0);
            tma_B(nxt);
          }
      } else {
      for (uint32_t it = 0; it < pre; ++it)
        asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(su32(&full[it])) : "memory");
      for (uint32_t nxt = NST; nxt < nkl; ++nxt) {
        const uint32_t s = nxt % NST;
        if (spin) mbar_wait_spin(&empty[s], ((nxt / NST) & 1) ^ 1);
        else mbar_wait(&empty[s], ((nxt / NST) & 1) ^ 1);   // MMA of stage nxt - NST retired
        if (t == 0) {
          mbar_arrive_tx(&full[s], abytes);
          tma_load_2d(sA + s * ABY, &wmap, &full[s], (int)((kb0 + nxt) * TC_BK), (int)m0);
        }
        issue_B(nxt, true);
      }
      }
    } else {
      // prologue path: wait for this thread's own copies of stage it (cp.async groups,
      // STAGES in flight), transform them in place, publish to the async proxy, arrive
      for (uint32_t it = 0; it < nkl; ++it) {
        const uint32_t issued = min(nkl, it + NST);
        switch (issued - it - 1) {
          case 0: cp_async_wait<0>(); break;
          case 1: cp_async_wait<1>(); break;
          case 2: cp_async_wait<2>(); break;
          default: cp_async_wait<3>(); break;
        }
        transform_B(it);
        fence_proxy_async();
        mbar_arrive(&full[it % NST]);
        const uint32_t nxt = it + NST;
        if (nxt < nkl) {
          const uint32_t s = nxt % NST;
          mbar_wait(&empty[s], ((nxt / NST) & 1) ^ 1);
          if (t == 0) {
            mbar_arrive_tx(&full[s], abytes);
            tma_load_2d(sA + s * ABY, &wmap, &full[s], (int)((kb0 + nxt) * TC_BK), (int)m0);
          }
          issue_B(nxt, false);
          cp_async_commit();
        }
      }
    }
  } else if (warp == 4) {
    // ------------------------------------------------------------ MMA warp
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(su32(tmem_slot)),
                 "r"(BN * TC_ACCS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    tc_fence_before();
    __syncwarp();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    if (lane == 0) {
      constexpr uint32_t IDESC = idesc_bf16(BM, BN);
      for (uint32_t it = 0; it < nkl; ++it) {
        const uint32_t s = it % NST;
        if (spin) mbar_wait_spin(&full[s], (it / NST) & 1);
        else mbar_wait(&full[s], (it / NST) & 1);
        if (trace && it == 0) tr[2] = globaltimer();
        fence_proxy_async();   // the gathered B tile was written through the generic proxy
        tc_fence_after();
        const uint32_t abase = su32(sA + s * ABY), bbase = su32(sB + s * BNB);
#pragma unroll
        for (uint32_t kk = 0; kk < TC_BK / 16; ++kk) {
          // TC_ACCS > 1: k-block it accumulates into accumulator it % TC_ACCS (independent
          // accumulation chains), summed by the epilogue
          umma_bf16(tmem + (it % TC_ACCS) * BN, sdesc_sw128(abase + kk * 32), sdesc_sw128(bbase + kk * 32), IDESC,
                    ((it / TC_ACCS) | kk) != 0 ? 1u : 0u);
        }
        umma_commit(&empty[s]);
      }
      umma_commit(accb);   // also orders the TMEM address write before the epilogue's read
      if (trace) tr[3] = globaltimer();
    }
    __syncwarp();
  }

  // ---------------------------------------------------------------- epilogue
  // 1. TMEM -> registers (warp w owns lanes = output channels 32w..32w+31) -> fp32
  //    tile in shared memory [pixel][channel] (conflict-free: a warp writes 32
  //    consecutive words of one pixel row)
  // every input of this block has been consumed: let the dependent kernel be placed
  // (its prologue overlaps this epilogue); warp 5 follows the accumulator too
  if (warp == 5 && nkl > 0) mbar_wait(accb, 0);
  constexpr uint32_t RELAXED_CTR = INSTR_CTR | INSTR_RELAXED;
  pdl_trigger();
  if constexpr (INSTR) {
    // relaxed exit count (B200-Q7): it orders nothing, so the bookkeeping warp
    // counts the block as soon as its MMAs are complete -- the count travels while the
    // epilogue runs instead of trailing the block's last store
    if (warp == 5 && lane == 0 && (ia.flags & RELAXED_CTR) == RELAXED_CTR)
      asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" ::"l"(ctr_of_block(ia) + 1) : "memory");
  }
  if (warp < 4) {
    // M = 128: accumulator row r in TMEM lane r (warp w reads lanes 32w..32w+31).  M = 64:
    // rows 16w..16w+15 in lanes 32w..32w+15 of each sub-partition (CUTLASS tmem_frg_1sm,
    // M_MMA = 64); the other half of the warp's lanes holds no row
    const uint32_t row = BM == 128 ? warp * 32 + lane : warp * 16 + (lane & 15);
    const bool owns = BM == 128 || lane < 16;
    if (nkl > 0) {
      mbar_wait(accb, 0);
      if (trace && threadIdx.x == 0) tr[4] = globaltimer();
      tc_fence_after();
      const uint32_t taddr = *tmem_slot + ((warp * 32) << 16);
#pragma unroll
      for (uint32_t c = 0; c < BN / 16; ++c) {
        float v[16];
        tmem_ld16(taddr + c * 16, v);
#pragma unroll
        for (uint32_t q = 1; q < TC_ACCS; ++q)
          if (q < nkl) {
            float u[16];
            tmem_ld16(taddr + q * BN + c * 16, u);
#pragma unroll
            for (int i = 0; i < 16; ++i) v[i] += u[i];
          }
#pragma unroll
        for (int i = 0; i < 16; ++i)
          if (owns) stage[(c * 16 + i) * BM + row] = v[i];
      }
      if (trace && threadIdx.x == 0) tr[8] = globaltimer();
    } else {
#pragma unroll 8
      for (uint32_t j = 0; j < BN; ++j)
        if (owns) stage[j * BM + row] = 0.f;
    }
  }
  if (a.ksplit == 1) {
    // 2. coalesced epilogue: item = (pixel, 8-channel group), 16-byte loads/stores
    if (warp < 4) {
      const uint32_t g = eg, co = eco;
      if (trace && threadIdx.x == 0) tr[9] = globaltimer();
      asm volatile("bar.sync 1, 128;" ::: "memory");   // the 4 epilogue warps only
      if (trace && threadIdx.x == 0) tr[10] = globaltimer();
      if (co < a.cout) {
        const bool rf = (a.flags & LF_RESIDUAL) != 0;
        if (a.act == 1) {
          if (rf) epi_tile<1, true, NIT, BM>(a, stage, n0, P, g, co, ebias, eres);
          else epi_tile<1, false, NIT, BM>(a, stage, n0, P, g, co, ebias, eres);
        } else if (a.act == 2) {
          if (rf) epi_tile<2, true, NIT, BM>(a, stage, n0, P, g, co, ebias, eres);
          else epi_tile<2, false, NIT, BM>(a, stage, n0, P, g, co, ebias, eres);
        } else {
          if (rf) epi_tile<0, true, NIT, BM>(a, stage, n0, P, g, co, ebias, eres);
          else epi_tile<0, false, NIT, BM>(a, stage, n0, P, g, co, ebias, eres);
        }
      }
    }
  } else if (!(a.flags & LF_SPLIT_DSMEM)) {
    // split-K across the CTAs of a cluster (1 x 1 x ksplit), reduced in L2: every CTA
    // adds its staged partial tile (only the rows holding pixels) into the tile's fp32
    // workspace with ONE bulk reduction (cp.reduce.async.bulk .add.f32: the adds run in
    // the L2, the SM streams the tile out at its store bandwidth instead of pushing it
    // over DSMEM at ~20 B/cycle and summing ks slices itself); after one cluster barrier
    // CTA r reads the sums of its 1/ksplit slice of pixel rows from L2, writes zeros back
    // (the workspace is all zero between launches) and runs the epilogue for them.  The
    // fp32 additions happen in L2 in arrival order (one bf16 rounding afterwards).
    // Items of thread t: pixel rows px0 + (t + 128 i) / 16 (i < 4), channel group t % 16.
    constexpr uint32_t MAXI = BN * (BM / 8) / (2 * NPROD);   // 4 items at ksplit 2 (BN 64)
    const uint32_t ks = a.ksplit;
    const uint32_t rows = BN / ks;
    const uint32_t px0 = split * rows;
    const uint32_t g = threadIdx.x % (BM / 8), co = m0 + g * 8;
    const uint32_t nitems = rows * (BM / 8);
    const uint32_t rv = n0 >= P ? 0u : min(BN, P - n0);   // pixel rows of the tile that exist
    float* wt = a.ws + (size_t)(tile_m * gridDim.x + tile_n) * (BN * BM);
    float bias[8];
    uint4 rres[MAXI];
    if (warp < 4 && co < a.cout) {
      load_bias8(a, co, bias);
      if (a.flags & LF_RESIDUAL) {
#pragma unroll
        for (uint32_t i = 0; i < MAXI; ++i) {
          const uint32_t item = threadIdx.x + i * NPROD;
          const uint32_t p = n0 + px0 + item / (BM / 8);
          if (item < nitems && p < P) rres[i] = load_res8(a, p, co);
        }
      }
    }
    if (warp < 4) {
      fence_proxy_async();                                 // staged rows -> the async proxy
      asm volatile("bar.sync 1, 128;" ::: "memory");      // all 4 staging warps are done
      if (threadIdx.x == 0 && nkl > 0 && rv > 0) {
        // rotated by the CTA's own slice (two bulk ranges) so that the ks CTAs of the
        // cluster start on different L2 lines instead of all adding into row 0 first
        const uint32_t r0 = (a.flags & LF_SPLIT_NOROT) ? 0u : min(px0, rv);
        const uint32_t sb = su32(stage);
        if (rv > r0)
          asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f32 [%0], [%1], %2;" ::"l"(
                           wt + r0 * BM),
                       "r"(sb + r0 * BM * 4), "r"((rv - r0) * BM * 4)
                       : "memory");
        if (r0 > 0)
          asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f32 [%0], [%1], %2;" ::"l"(wt),
                       "r"(sb), "r"(r0 * BM * 4)
                       : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");   // the adds are performed
        asm volatile("fence.proxy.async.global;" ::: "memory");      // ... before the generic release
        if (!(a.flags & LF_SPLIT_RELBAR)) asm volatile("fence.acq_rel.cluster;" ::: "memory");
      }
    }
    if (trace && threadIdx.x == 0) tr[9] = globaltimer();
    __syncwarp();
    // every CTA's additions are complete and visible cluster-wide: the one thread that
    // issued them released them with its fence; the barrier then only needs to order
    // (relaxed arrive) and every reader acquires after it
    if (a.flags & LF_SPLIT_RELBAR)
      asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    else
      asm volatile("barrier.cluster.arrive.relaxed.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    if (trace && threadIdx.x == 0) tr[10] = globaltimer();
    if (warp < 4 && co < a.cout) {
#pragma unroll
      for (uint32_t i = 0; i < MAXI; ++i) {
        const uint32_t item = threadIdx.x + i * NPROD;
        const uint32_t r = item / (BM / 8), p = n0 + px0 + r;
        if (item < nitems && p < P) {
          float* q = wt + (px0 + r) * BM + g * 8;
          float v[8];
          asm volatile("ld.relaxed.gpu.global.L1::no_allocate.v4.f32 {%0, %1, %2, %3}, [%4];"
                       : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3])
                       : "l"(q));
          asm volatile("ld.relaxed.gpu.global.L1::no_allocate.v4.f32 {%0, %1, %2, %3}, [%4];"
                       : "=f"(v[4]), "=f"(v[5]), "=f"(v[6]), "=f"(v[7])
                       : "l"(q + 4));
          asm volatile("st.global.v4.f32 [%0], {%1, %1, %1, %1};\n\tst.global.v4.f32 [%2], {%1, %1, %1, %1};" ::"l"(q),
                       "f"(0.f), "l"(q + 4)
                       : "memory");
          epi_store8(a, p, co, v, bias, rres[i]);
        }
      }
      fence_proxy_async_global();   // the zeros, before a later grid's bulk reductions
    }
    if (trace && threadIdx.x == 0) tr[14] = globaltimer();
  } else {
    // (A/B, LF_SPLIT_DSMEM) split-K across the CTAs of a cluster (1 x 1 x ksplit): CTA r owns a 1/ksplit
    // slice of the tile's pixel rows.  Every CTA PUSHES the other slices of its staged
    // partial tile to their owners with one bulk DSMEM copy each (cp.async.bulk
    // shared::cta -> shared::cluster, completing on the owner's mbarrier); the owner
    // sums its slice and the ks - 1 received ones from local shared memory and runs the
    // epilogue for it -- no global workspace, no atomics, no per-element remote loads
    // (those were bound at ~17 GB/s per SM: 1.7 us for ksplit 8).
    // Items of thread t: pixel rows px0 + (t + 128 i) / 16 (i < 4), channel group t % 16.
    constexpr uint32_t MAXI = BN * (BM / 8) / (2 * NPROD);   // 4 items at ksplit 2 (BN 64)
    const uint32_t ks = a.ksplit;
    const uint32_t rows = BN / ks;
    const uint32_t px0 = split * rows;
    const uint32_t g = threadIdx.x % (BM / 8), co = m0 + g * 8;
    const uint32_t nitems = rows * (BM / 8);
    const uint32_t slice = rows * BM * 4;                // bytes of one slice (slot pitch)
    float* recv = stage + BN * BM;                       // ks - 1 received slices (free A stages)
    // only the slice rows that hold real pixels travel (the tile tail past P does not)
    auto valid_rows = [&](uint32_t owner) -> uint32_t {
      const uint32_t r0 = n0 + owner * rows;
      return r0 >= P ? 0u : min(rows, P - r0);
    };
    float bias[8];
    uint4 rres[MAXI];
    if (warp < 4 && co < a.cout) {
      load_bias8(a, co, bias);
      if (a.flags & LF_RESIDUAL) {
#pragma unroll
        for (uint32_t i = 0; i < MAXI; ++i) {
          const uint32_t item = threadIdx.x + i * NPROD;
          const uint32_t p = n0 + px0 + item / (BM / 8);
          if (item < nitems && p < P) rres[i] = load_res8(a, p, co);
        }
      }
    }
    if (threadIdx.x == 0) mbar_arrive_tx(rbar, (ks - 1) * valid_rows(split) * BM * 4);   // before any push
    if (warp < 4) fence_proxy_async();   // the staged tile (generic writes) is read by the bulk copies
    __syncwarp();
    if (trace && threadIdx.x == 0) tr[9] = globaltimer();
    // every CTA's staged tile and armed barrier are visible cluster-wide (restricted
    // release fence: MEMBAR.CTA, not MEMBAR.GPU), then a relaxed arrive
    asm volatile(
        "fence.release.sync_restrict::shared::cta.cluster;\n\t"
        "barrier.cluster.arrive.relaxed.aligned;\n\tbarrier.cluster.wait.aligned;" ::: "memory");
    if (trace && threadIdx.x == 0) tr[10] = globaltimer();
    if (threadIdx.x == 0) {
      // staggered: CTA r sends to r + 1, r + 2, ...; the slot in the owner's buffer is
      // the sender's distance behind it
      for (uint32_t j = 1; j < ks; ++j) {
        const uint32_t owner = (split + j) & (ks - 1);
        const uint32_t bytes = valid_rows(owner) * BM * 4;
        if (bytes == 0) continue;
        const uint32_t slot = (split + ks - owner - 1) & (ks - 1);
        uint32_t dst, bar;
        asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(dst) : "r"(su32(recv) + slot * slice), "r"(owner));
        asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(bar) : "r"(su32(rbar)), "r"(owner));
        asm volatile(
            "cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
            "r"(su32(stage) + owner * slice), "r"(bytes), "r"(bar)
            : "memory");
      }
    }
    if (warp < 4 && co < a.cout) {
      mbar_wait(rbar, 0);   // the ks - 1 slices of our rows have landed
      if (trace && threadIdx.x == 0) tr[15] = globaltimer();
#pragma unroll
      for (uint32_t i = 0; i < MAXI; ++i) {
        const uint32_t item = threadIdx.x + i * NPROD;
        const uint32_t r = item / (BM / 8), p = n0 + px0 + r;
        if (item < nitems && p < P) {
          const float4* own = reinterpret_cast<const float4*>(stage + (px0 + r) * BM + g * 8);
          float4 x0 = own[0], x1 = own[1];
          for (uint32_t q = 0; q + 1 < ks; ++q) {
            const float4* o = reinterpret_cast<const float4*>(recv + (q * rows + r) * BM + g * 8);
            const float4 y0 = o[0], y1 = o[1];
            x0.x += y0.x; x0.y += y0.y; x0.z += y0.z; x0.w += y0.w;
            x1.x += y1.x; x1.y += y1.y; x1.z += y1.z; x1.w += y1.w;
          }
          const float v[8] = {x0.x, x0.y, x0.z, x0.w, x1.x, x1.y, x1.z, x1.w};
          epi_store8(a, p, co, v, bias, rres[i]);
        }
      }
    }
    // no CTA may leave while a peer still reads its shared memory
    if (trace && threadIdx.x == 0) tr[14] = globaltimer();
    __syncwarp();
    asm volatile("barrier.cluster.arrive.relaxed.aligned;\n\tbarrier.cluster.wait.aligned;" ::: "memory");
  }
  if (trace && threadIdx.x == 0) tr[5] = globaltimer();
  tc_fence_before();
  __syncthreads();
  if (warp == 4) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(*tmem_slot), "r"(BN * TC_ACCS) : "memory");
    // every other thread is past the barrier above: the MMA warp, last to finish, counts
    // the block's exit itself (no second block barrier)
    if (trace && lane == 0) tr[6] = globaltimer();
    if (lane == 0 && (ia.flags & RELAXED_CTR) != RELAXED_CTR) instr_exit_last_thread<INSTR>(ia);
    if (trace && lane == 0) tr[7] = globaltimer();
  }
}

uint32_t tc_smem_bytes() { return 1024 + TC_RING + 512; }   // align pad + stage ring + barriers
static_assert(TC_RING == TC_STAGES * (A_BYTES + B_BYTES), "ring");

void tc_kernel_table(KernelFn* instr, KernelFn* plain) {
  instr[0] = (KernelFn)k_conv_tc<true, false, TC_BN>;
  plain[0] = (KernelFn)k_conv_tc<false, false, TC_BN>;
  instr[1] = (KernelFn)k_conv_tc<true, true, TC_BN>;     // with the DenseNet prologue
  plain[1] = (KernelFn)k_conv_tc<false, true, TC_BN>;
  instr[2] = (KernelFn)k_conv_tc<true, false, TC_BN_WIDE>;   // 128-pixel tiles
  plain[2] = (KernelFn)k_conv_tc<false, false, TC_BN_WIDE>;
  instr[3] = (KernelFn)k_conv_tc<true, false, TC_BN, 64>;    // narrow layers: UMMA M = 64
  plain[3] = (KernelFn)k_conv_tc<false, false, TC_BN, 64>;
}

// Host: tensor map for the packed weights [rows][kpad] bf16, box 64 x box_rows
// (128, or Cout rounded up to 8 for narrow layers), SW128.
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int make_weight_tmap(void* weights, uint32_t rows, uint32_t kpad, uint32_t box_rows, void* out128) {
  static EncodeTiledFn enc = nullptr;
  if (!enc) {
    cudaDriverEntryPointQueryResult q;
    void* fn = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !fn)
      return -1;
    enc = (EncodeTiledFn)fn;
  }
  cuuint64_t dims[2] = {kpad, rows};
  cuuint64_t strides[1] = {(cuuint64_t)kpad * 2};
  cuuint32_t box[2] = {TC_BK, box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = enc((CUtensorMap*)out128, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, weights, dims, strides, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? 0 : -1;
}


// Host: im2col tensor map of a conv's NHWC bf16 input (batch 1) for LF_TMA_B: channels
// [in_co, in_co + cin) of a buffer with channel stride in_cs, BN pixels x 64 channels per
// load, SW128 (the B operand's K-major layout), conv strides as traversal strides, the
// padded window range as the pixel bounding box (out of bounds -> zero = padding).
typedef CUresult (*EncodeIm2colFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const int*, const int*, cuuint32_t, cuuint32_t,
                                   const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                   CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int make_im2col_tmap(const void* in, const LayerArgs& a, uint32_t bn, void* out128) {
  static EncodeIm2colFn enc = nullptr;
  if (!enc) {
    cudaDriverEntryPointQueryResult q;
    void* fn = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeIm2col", &fn, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !fn)
      return -1;
    enc = (EncodeIm2colFn)fn;
  }
  const cuuint64_t px = (cuuint64_t)a.in_cs * 2;
  cuuint64_t dims[4] = {a.cin, a.w_, a.h, 1};
  cuuint64_t strides[3] = {px, px * a.w_, px * a.w_ * a.h};
  int lower[2] = {-(int)a.pw, -(int)a.ph};                                     // {W, H}
  int upper[2] = {(int)a.pw - ((int)a.kw - 1), (int)a.ph - ((int)a.kh - 1)};
  cuuint32_t estr[4] = {1, a.sw, a.sh, 1};
  CUresult r = enc((CUtensorMap*)out128, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4,
                   (void*)((const uint8_t*)in + (size_t)a.in_co * 2), dims, strides, lower, upper, TC_BK, bn, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? 0 : -1;
}

}  // namespace paella
