// SIMT inference kernels (K2b-K2e, and the fp32 / fallback-free SIMT conv K2a-simt).
//
// All activations are NHWC with an explicit channel stride (LayerArgs::*_cs) and
// channel offset (*_co): channel counts are multiples of 8 after the ingest pads the
// image to 8 channels, so every thread moves 8 channels = one 16-byte vector (bf16)
// or two (fp32).  Every kernel is built twice (INSTR = true: Paella-instrumented,
// false: the uninstrumented twin used by the naive baseline and the overhead
// microbenchmark).  No kernel returns early: instr_exit needs every thread.
#include <cuda_bf16.h>

#include "common.h"
#include "instr.cuh"
#include "kernels.h"

namespace paella {

// ---------------------------------------------------------------------------
// 8-element vector load / store
// ---------------------------------------------------------------------------
__device__ __forceinline__ void load8(const __nv_bfloat16* p, float (&v)[8]) {
  uint4 u = *reinterpret_cast<const uint4*>(p);
  const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    float2 f = __bfloat1622float2(h[i]);
    v[2 * i] = f.x;
    v[2 * i + 1] = f.y;
  }
}
__device__ __forceinline__ void load8(const float* p, float (&v)[8]) {
  float4 a = reinterpret_cast<const float4*>(p)[0];
  float4 b = reinterpret_cast<const float4*>(p)[1];
  v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
  v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
}
__device__ __forceinline__ void store8(__nv_bfloat16* p, const float (&v)[8]) {
  uint4 u;
  __nv_bfloat162* h = reinterpret_cast<__nv_bfloat162*>(&u);
#pragma unroll
  for (int i = 0; i < 4; ++i) h[i] = __floats2bfloat162_rn(v[2 * i], v[2 * i + 1]);  // RNE
  *reinterpret_cast<uint4*>(p) = u;
}
__device__ __forceinline__ void store8(float* p, const float (&v)[8]) {
  reinterpret_cast<float4*>(p)[0] = make_float4(v[0], v[1], v[2], v[3]);
  reinterpret_cast<float4*>(p)[1] = make_float4(v[4], v[5], v[6], v[7]);
}

__device__ __forceinline__ float act_f(float x, uint32_t act) {
  if (act == 1) return fmaxf(x, 0.f);
  if (act == 2) return fminf(fmaxf(x, 0.f), 6.f);
  return x;
}

// ---------------------------------------------------------------------------
// K2e ingest: client fp32 NCHW (pinned, mapped host memory) -> model dtype NHWC,
// channels padded to 8 with zeros.  bf16 rounding is RNE (reading C1-Q7).
// ---------------------------------------------------------------------------
template <typename T, bool INSTR>
__global__ void __launch_bounds__(256) k_ingest(const __grid_constant__ LayerArgs a,
                                                const __grid_constant__ InstrArgs ia) {
  kernel_begin<INSTR>(ia);
  const float* in = static_cast<const float*>(a.in);
  T* out = static_cast<T*>(a.out);
  uint32_t hw = a.h * a.w_;
  if ((hw & 3) == 0 && (reinterpret_cast<uintptr_t>(in) & 15) == 0) {
    // 4 consecutive pixels per thread: one 16-byte read per channel plane (fewer,
    // larger PCIe read requests), four 16-byte NHWC stores
    const uint32_t p = 4 * (blockIdx.x * blockDim.x + threadIdx.x);
    if (p < hw) {
      float4 q[8];
#pragma unroll
      for (int c = 0; c < 8; ++c)
        q[c] = (c < (int)a.cin) ? __ldcs(reinterpret_cast<const float4*>(in + (size_t)c * hw + p))
                                : make_float4(0.f, 0.f, 0.f, 0.f);
      float v[4][8];
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        v[0][c] = q[c].x;
        v[1][c] = q[c].y;
        v[2][c] = q[c].z;
        v[3][c] = q[c].w;
      }
#pragma unroll
      for (int i = 0; i < 4; ++i) store8(out + (size_t)(p + i) * a.out_cs + a.out_co, v[i]);
    }
  } else {
    uint32_t p = blockIdx.x * blockDim.x + threadIdx.x;
    for (; p < hw; p += gridDim.x * blockDim.x) {
      float v[8];
#pragma unroll
      for (int c = 0; c < 8; ++c) v[c] = (c < (int)a.cin) ? __ldcs(in + (size_t)c * hw + p) : 0.f;
      store8(out + (size_t)p * a.out_cs + a.out_co, v);
    }
  }
  instr_exit<INSTR>(ia);
}

// ---------------------------------------------------------------------------
// K2a (SIMT): conv as implicit GEMM  D[Cout x P] = W[Cout x K] . im2col(X)[K x P],
// K = kh*kw*cin ordered (r, s, ci) so 8 consecutive k are 8 consecutive channels.
// Tile 64 (cout) x 64 (pixels) x 32 (k), 256 threads, 4x4 outputs per thread.
// Weights packed [cout][Kpad] (Kpad = K rounded up to 64, zero-filled).
// Used for the fp32 path (SIMT FFMA, no TF32 -- reading C1-Q3) and for convs the
// tcgen05 kernel does not take.  Epilogue: bias, residual (fp32), activation, one
// rounding.
// ---------------------------------------------------------------------------
template <typename T, bool INSTR>
__global__ void __launch_bounds__(256) k_conv_simt(const __grid_constant__ LayerArgs a,
                                                   const __grid_constant__ InstrArgs ia) {
  kernel_begin<INSTR>(ia);
  constexpr int BM = 64, BN = 64, BK = 32;
  __shared__ float As[BK][BM + 4];
  __shared__ float Bs[BK][BN + 4];
  const T* X = static_cast<const T*>(a.in);
  const T* W = static_cast<const T*>(a.w);
  const int tid = threadIdx.x;
  const int co0 = blockIdx.y * BM;
  const int p0 = blockIdx.x * BN;
  const int P = a.oh * a.ow;
  const int K = a.kh * a.kw * a.cin;
  const int tm = tid % 16, tn = tid / 16;
  float acc[4][4];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;

  // this thread's B-load pixel
  const int lp = tid % 64, lkg = tid / 64;   // pixel, k-granule (0..3)
  const int gp = p0 + lp;
  const int oh = gp / a.ow, ow = gp % a.ow;
  // this thread's A-load row
  const int arow = tid / 4, akg = tid % 4;

  for (int k0 = 0; k0 < (int)a.kpad; k0 += BK) {
    {  // A: 64 rows x 32 k
      float v[8];
      int co = co0 + arow;
      if (co < (int)a.cout) {
        load8(W + (size_t)co * a.kpad + k0 + akg * 8, v);
      } else {
#pragma unroll
        for (int i = 0; i < 8; ++i) v[i] = 0.f;
      }
#pragma unroll
      for (int i = 0; i < 8; ++i) As[akg * 8 + i][arow] = v[i];
    }
    {  // B: 32 k x 64 pixels, im2col gather
      float v[8];
      int k = k0 + lkg * 8;
      bool ok = (gp < P) && (k < K);
      int ci = 0, ih = 0, iw = 0;
      if (ok) {
        ci = k % a.cin;
        int rs = k / a.cin;
        int s = rs % a.kw, r = rs / a.kw;
        ih = oh * a.sh - a.ph + r;
        iw = ow * a.sw - a.pw + s;
        ok = ih >= 0 && ih < (int)a.h && iw >= 0 && iw < (int)a.w_;
      }
      if (ok) {
        load8(X + ((size_t)ih * a.w_ + iw) * a.in_cs + a.in_co + ci, v);
        if (a.flags & LF_PROLOGUE) {
#pragma unroll
          for (int i = 0; i < 8; ++i) v[i] = fmaxf(fmaf(a.pro_scale[ci + i], v[i], a.pro_shift[ci + i]), 0.f);
        }
      } else {
#pragma unroll
        for (int i = 0; i < 8; ++i) v[i] = 0.f;
      }
#pragma unroll
      for (int i = 0; i < 8; ++i) Bs[lkg * 8 + i][lp] = v[i];
    }
    __syncthreads();
#pragma unroll 8
    for (int k = 0; k < BK; ++k) {
      float4 av = *reinterpret_cast<const float4*>(&As[k][tm * 4]);
      float4 bv = *reinterpret_cast<const float4*>(&Bs[k][tn * 4]);
      float am[4] = {av.x, av.y, av.z, av.w};
      float bn[4] = {bv.x, bv.y, bv.z, bv.w};
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(am[i], bn[j], acc[i][j]);
    }
    __syncthreads();
  }
  // epilogue
  T* Y = static_cast<T*>(a.out);
  const T* Rz = static_cast<const T*>(a.res);
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    int p = p0 + tn * 4 + j;
    if (p >= P) continue;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      int co = co0 + tm * 4 + i;
      if (co >= (int)a.cout) continue;
      float v = acc[i][j] + a.bias[co];
      if (a.flags & LF_RESIDUAL) v += (float)Rz[(size_t)p * a.res_cs + a.res_co + co];
      v = act_f(v, a.act);
      Y[(size_t)p * a.out_cs + a.out_co + co] = (T)v;
    }
  }
  instr_exit<INSTR>(ia);
}

// ---------------------------------------------------------------------------
// K2c depthwise conv (groups == cin == cout).  One thread per (output pixel, 8-channel
// granule); for the 3x3 case (every depthwise layer of MobileNetV2) all 9 taps of
// activations and weights are loaded before any arithmetic so the 18 independent
// 16-byte loads are in flight together (latency, not bandwidth, bounds batch 1).
// Weights packed [kh][kw][c].
// ---------------------------------------------------------------------------
template <typename T, int KH, int KW>
__device__ __forceinline__ void dw_taps(const LayerArgs& a, const T* X, const T* W, int oh, int ow, int c,
                                        float (&acc)[8]) {
  float xv[KH * KW][8], wv[KH * KW][8];
#pragma unroll
  for (int r = 0; r < KH; ++r)
#pragma unroll
    for (int s = 0; s < KW; ++s) {
      const int ih = oh * (int)a.sh - (int)a.ph + r, iw = ow * (int)a.sw - (int)a.pw + s;
      const bool ok = ih >= 0 && ih < (int)a.h && iw >= 0 && iw < (int)a.w_;
      if (ok) {
        load8(X + ((size_t)ih * a.w_ + iw) * a.in_cs + a.in_co + c, xv[r * KW + s]);
      } else {
#pragma unroll
        for (int i = 0; i < 8; ++i) xv[r * KW + s][i] = 0.f;
      }
      load8(W + ((size_t)r * KW + s) * a.cout + c, wv[r * KW + s]);
    }
#pragma unroll
  for (int t = 0; t < KH * KW; ++t)
#pragma unroll
    for (int i = 0; i < 8; ++i) acc[i] = fmaf(wv[t][i], xv[t][i], acc[i]);
}

template <typename T, bool INSTR>
__global__ void __launch_bounds__(256) k_dwconv(const __grid_constant__ LayerArgs a,
                                                const __grid_constant__ InstrArgs ia) {
  kernel_begin<INSTR>(ia);
  const T* X = static_cast<const T*>(a.in);
  const T* W = static_cast<const T*>(a.w);
  T* Y = static_cast<T*>(a.out);
  uint32_t ng = a.cout / 8;
  uint32_t idx = blockIdx.x * blockDim.x + threadIdx.x;
  uint32_t P = a.oh * a.ow;
  if (idx < P * ng) {
    uint32_t g = idx % ng, p = idx / ng;
    int oh = p / a.ow, ow = p % a.ow;
    int c = g * 8;
    float acc[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) acc[i] = a.bias[c + i];
    if (a.kh == 3 && a.kw == 3) {
      dw_taps<T, 3, 3>(a, X, W, oh, ow, c, acc);
    } else {
      for (int r = 0; r < (int)a.kh; ++r) {
        int ih = oh * a.sh - a.ph + r;
        if (ih < 0 || ih >= (int)a.h) continue;
        for (int s = 0; s < (int)a.kw; ++s) {
          int iw = ow * a.sw - a.pw + s;
          if (iw < 0 || iw >= (int)a.w_) continue;
          float xv[8], wv[8];
          load8(X + ((size_t)ih * a.w_ + iw) * a.in_cs + a.in_co + c, xv);
          load8(W + ((size_t)r * a.kw + s) * a.cout + c, wv);
#pragma unroll
          for (int i = 0; i < 8; ++i) acc[i] = fmaf(wv[i], xv[i], acc[i]);
        }
      }
    }
    if (a.flags & LF_RESIDUAL) {
      float rv[8];
      load8(static_cast<const T*>(a.res) + (size_t)p * a.res_cs + a.res_co + c, rv);
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] += rv[i];
    }
#pragma unroll
    for (int i = 0; i < 8; ++i) acc[i] = act_f(acc[i], a.act);
    store8(Y + (size_t)p * a.out_cs + a.out_co + c, acc);
  }
  instr_exit<INSTR>(ia);
}

// ---------------------------------------------------------------------------
// K2d pooling.  max: padding = -inf, ceil-mode windows clipped to the input;
// avg: count_include_pad (divisor k*k).  One thread per (pixel, granule); square
// 2x2 / 3x3 windows load every tap before reducing (independent loads in flight).
// ---------------------------------------------------------------------------
template <typename T, bool MAX, int K>
__device__ __forceinline__ void pool_taps(const LayerArgs& a, const T* X, int oh, int ow, int c, float (&acc)[8]) {
  float xv[K * K][8];
  bool ok[K * K];
#pragma unroll
  for (int r = 0; r < K; ++r)
#pragma unroll
    for (int s = 0; s < K; ++s) {
      const int ih = oh * (int)a.sh - (int)a.ph + r, iw = ow * (int)a.sw - (int)a.pw + s;
      ok[r * K + s] = ih >= 0 && ih < (int)a.h && iw >= 0 && iw < (int)a.w_;
      if (ok[r * K + s]) load8(X + ((size_t)ih * a.w_ + iw) * a.in_cs + a.in_co + c, xv[r * K + s]);
    }
#pragma unroll
  for (int t = 0; t < K * K; ++t)
    if (ok[t]) {
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] = MAX ? fmaxf(acc[i], xv[t][i]) : acc[i] + xv[t][i];
    }
}

template <typename T, bool INSTR, bool MAX>
__global__ void __launch_bounds__(256) k_pool(const __grid_constant__ LayerArgs a,
                                              const __grid_constant__ InstrArgs ia) {
  kernel_begin<INSTR>(ia);
  const T* X = static_cast<const T*>(a.in);
  T* Y = static_cast<T*>(a.out);
  uint32_t ng = a.cout / 8;
  uint32_t idx = blockIdx.x * blockDim.x + threadIdx.x;
  uint32_t P = a.oh * a.ow;
  if (idx < P * ng) {
    uint32_t g = idx % ng, p = idx / ng;
    int oh = p / a.ow, ow = p % a.ow;
    int c = g * 8;
    float acc[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) acc[i] = MAX ? -INFINITY : 0.f;
    if (a.kh == 3 && a.kw == 3) {
      pool_taps<T, MAX, 3>(a, X, oh, ow, c, acc);
    } else if (a.kh == 2 && a.kw == 2) {
      pool_taps<T, MAX, 2>(a, X, oh, ow, c, acc);
    } else {
      for (int r = 0; r < (int)a.kh; ++r) {
        int ih = oh * a.sh - a.ph + r;
        if (ih < 0 || ih >= (int)a.h) continue;
        for (int s = 0; s < (int)a.kw; ++s) {
          int iw = ow * a.sw - a.pw + s;
          if (iw < 0 || iw >= (int)a.w_) continue;
          float xv[8];
          load8(X + ((size_t)ih * a.w_ + iw) * a.in_cs + a.in_co + c, xv);
#pragma unroll
          for (int i = 0; i < 8; ++i) acc[i] = MAX ? fmaxf(acc[i], xv[i]) : acc[i] + xv[i];
        }
      }
    }
    if (!MAX) {
      float inv = 1.f / (float)(a.kh * a.kw);
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] *= inv;
    }
    store8(Y + (size_t)p * a.out_cs + a.out_co + c, acc);
  }
  instr_exit<INSTR>(ia);
}

// ---------------------------------------------------------------------------
// Global average pool (+ optional DenseNet prologue).  8 threads per 8-channel
// granule split the pixels and reduce with shuffles; the output is either an
// activation (C,1,1) or, if final, fp32 logits in client memory.
// ---------------------------------------------------------------------------
template <typename T, bool INSTR>
__global__ void __launch_bounds__(256) k_gap(const __grid_constant__ LayerArgs a,
                                             const __grid_constant__ InstrArgs ia) {
  kernel_begin<INSTR>(ia);
  const T* X = static_cast<const T*>(a.in);
  uint32_t ng = a.cout / 8;
  uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
  uint32_t g = tid / 32, l = tid % 32;   // a warp per 8-channel granule
  float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  const uint32_t HW = a.h * a.w_;
  if (g < ng) {
    int c = g * 8;
    float sc[8], sh[8];
    if (a.flags & LF_PROLOGUE) {
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        sc[i] = a.pro_scale[c + i];
        sh[i] = a.pro_shift[c + i];
      }
    }
#pragma unroll 4
    for (uint32_t p = l; p < HW; p += 32) {
      float xv[8];
      load8(X + (size_t)p * a.in_cs + a.in_co + c, xv);
      if (a.flags & LF_PROLOGUE) {
#pragma unroll
        for (int i = 0; i < 8; ++i) xv[i] = fmaxf(fmaf(sc[i], xv[i], sh[i]), 0.f);
      }
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] += xv[i];
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1)
#pragma unroll
    for (int i = 0; i < 8; ++i) acc[i] += __shfl_xor_sync(0xffffffffu, acc[i], o);
  if (g < ng && l == 0) {
    int c = g * 8;
    float inv = 1.f / (float)HW;
#pragma unroll
    for (int i = 0; i < 8; ++i) acc[i] *= inv;
    if (a.flags & LF_FINAL) {
      store8(static_cast<float*>(a.out) + c, acc);
    } else {
      store8(static_cast<T*>(a.out) + a.out_co + c, acc);
    }
  }
  instr_exit<INSTR>(ia);
}

// ---------------------------------------------------------------------------
// K2b FC at batch 1 = weight-streaming GEMV (HBM-bound: no tensor cores, reading of
// the north star "do not reshape HBM-bound work into GEMMs").  One warp per output
// row, 16-byte weight loads, fp32 accumulate, warp-shuffle reduction.  Weights
// [cout][kpad] in NHWC-flatten order (the planner permutes torch's NCHW flatten).
// ---------------------------------------------------------------------------
template <typename T, bool INSTR>
__global__ void __launch_bounds__(256) k_fc(const __grid_constant__ LayerArgs a,
                                            const __grid_constant__ InstrArgs ia) {
  kernel_begin<INSTR>(ia);
  const T* X = static_cast<const T*>(a.in);
  const T* W = static_cast<const T*>(a.w);
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int row = blockIdx.x * 8 + warp;
  const int K = a.cin;   // multiple of 8, input contiguous (checked by the planner)
  if (row < (int)a.cout) {
    float acc = 0.f;
    const T* wr = W + (size_t)row * a.kpad;
    for (int k = lane * 8; k < K; k += 32 * 8) {
      float wv[8], xv[8];
      load8(wr + k, wv);
      load8(X + a.in_co + k, xv);
#pragma unroll
      for (int i = 0; i < 8; ++i) acc = fmaf(wv[i], xv[i], acc);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0) {
      float v = act_f(acc + a.bias[row], a.act);
      if (a.flags & LF_FINAL)
        static_cast<float*>(a.out)[row] = v;
      else
        static_cast<T*>(a.out)[a.out_co + row] = (T)v;
    }
  }
  instr_exit<INSTR>(ia);
}

// ---------------------------------------------------------------------------
// Fused global-average-pool + FC (the classifier head of ResNet / MobileNetV2 /
// DenseNet / Inception): one launch instead of two.  Every block (32 output rows)
// first averages the C x HW input into shared memory (+ DenseNet's norm5 prologue),
// then each warp streams 4 weight rows against it.  Same arithmetic and rounding
// points as GAP -> FC except that the pooled vector stays fp32 (no bf16 rounding
// between the two, reading C1-Q7: one rounding per fused layer).
// ---------------------------------------------------------------------------
template <typename T, bool INSTR>
__global__ void __launch_bounds__(256) k_gapfc(const __grid_constant__ LayerArgs a,
                                                  const __grid_constant__ InstrArgs ia) {
  // Batch-1 latency layout: clusters of GAPFC_CLUSTER CTAs; the CTAs of a cluster
  // pool 1/GAPFC_CLUSTER of the channels each, exchange the pooled slices over DSMEM,
  // then every warp computes one FC row (8 rows per CTA, ~128 CTAs for 1000 classes:
  // the weight stream is spread over many SMs).  Latency (phase traces, ResNet-50 head
  // in a PDL chain: pool 3.0 us, barrier + DSMEM gather 1.1 us, FC 1.4 us): every thread
  // issues all its pooling loads at once (pool 3.0 -> 2.1 us, last CTA exit 7.5 -> 6.7 us).
  // Prefetching the FC weight rows into registers before the PDL wait was measured
  // slower: the registers it needs keep the head's CTAs from co-residing with the
  // predecessor's, so they are placed later.
  const bool trace = (a.flags & LF_TRACE) != 0;   // debug: per-CTA phase timestamps (thread 0)
  uint64_t* tr = trace ? a.trace + 16 * blockIdx.x : nullptr;
  auto mark = [&](int k) {
    if (trace && threadIdx.x == 0) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tr[k]));
  };
  mark(0);
  instr_enter<INSTR>(ia);
  extern __shared__ float pooled[];   // [C], every CTA ends up with all of it
  const T* X = static_cast<const T*>(a.in);
  const T* W = static_cast<const T*>(a.w);
  const uint32_t C = a.cin, HW = a.h * a.w_, NG = C / 8;
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int row = blockIdx.x * (blockDim.x / 32) + warp;
  pdl_wait();
  pdl_trigger();
  mark(1);
  const float inv = 1.f / (float)HW;
  uint32_t rank;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
  const uint32_t per = (NG + GAPFC_CLUSTER - 1) / GAPFC_CLUSTER;   // granules per CTA
  const uint32_t g0 = rank * per, g1 = min(NG, g0 + per);
  uint32_t tpg = 32;
  while (tpg > 1 && per * tpg > blockDim.x) tpg >>= 1;
  const uint32_t sub = threadIdx.x % tpg, gpb = blockDim.x / tpg;
  for (uint32_t gi = threadIdx.x / tpg; gi < (per + gpb - 1) / gpb * gpb; gi += gpb) {
    const uint32_t g = g0 + gi;
    float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    if (g < g1) {
      const uint32_t c = g * 8;
      float sc[8], sh[8];
      if (a.flags & LF_PROLOGUE) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          sc[i] = a.pro_scale[c + i];
          sh[i] = a.pro_shift[c + i];
        }
      }
      const T* xp = X + a.in_co + c;
      constexpr uint32_t MAXL = 8;   // pooling loads per thread issued together (bf16: raw 16 B)
      if (sizeof(T) == 2 && HW <= MAXL * tpg) {
        uint4 raw[MAXL];
#pragma unroll
        for (uint32_t t = 0; t < MAXL; ++t) {
          const uint32_t p = sub + t * tpg;
          raw[t] = *reinterpret_cast<const uint4*>(xp + (size_t)(p < HW ? p : 0u) * a.in_cs);
        }
#pragma unroll
        for (uint32_t t = 0; t < MAXL; ++t) {
          if (sub + t * tpg < HW) {
            const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&raw[t]);
            float xv[8];
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              const float2 f = __bfloat1622float2(h[i]);
              xv[2 * i] = f.x;
              xv[2 * i + 1] = f.y;
            }
            if (a.flags & LF_PROLOGUE) {
#pragma unroll
              for (int i = 0; i < 8; ++i) xv[i] = fmaxf(fmaf(sc[i], xv[i], sh[i]), 0.f);
            }
#pragma unroll
            for (int i = 0; i < 8; ++i) acc[i] += xv[i];
          }
        }
      } else {
#pragma unroll 4
        for (uint32_t p = sub; p < HW; p += tpg) {
          float xv[8];
          load8(xp + (size_t)p * a.in_cs, xv);
          if (a.flags & LF_PROLOGUE) {
#pragma unroll
            for (int i = 0; i < 8; ++i) xv[i] = fmaxf(fmaf(sc[i], xv[i], sh[i]), 0.f);
          }
#pragma unroll
          for (int i = 0; i < 8; ++i) acc[i] += xv[i];
        }
      }
    }
    for (uint32_t o = tpg / 2; o > 0; o >>= 1)
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] += __shfl_xor_sync(0xffffffffu, acc[i], o);
    if (g < g1 && sub == 0) {
#pragma unroll
      for (int i = 0; i < 8; ++i) pooled[g * 8 + i] = acc[i] * inv;
    }
  }
  mark(2);
  // publish the slice to the cluster (restricted release: MEMBAR.CTA), then gather the
  // peers' slices (16-byte DSMEM loads) into the local copy
  asm volatile(
      "fence.release.sync_restrict::shared::cta.cluster;\n\t"
      "barrier.cluster.arrive.relaxed.aligned;\n\tbarrier.cluster.wait.aligned;" ::: "memory");
  mark(3);
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(pooled);
  for (uint32_t q = threadIdx.x; q < C / 4; q += blockDim.x) {
    const uint32_t owner = (q * 4 / 8) / per;
    if (owner == rank) continue;
    uint32_t peer;
    float4 v;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(peer) : "r"(base + q * 16), "r"(owner));
    asm volatile("ld.shared::cluster.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
                 : "r"(peer));
    reinterpret_cast<float4*>(pooled)[q] = v;
  }
  // done reading the peers; the matching wait (peers stay resident) is at the end
  asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");
  __syncthreads();
  mark(4);
  if (row < (int)a.cout) {
    const T* wr = W + (size_t)row * a.kpad;
    float acc = 0.f;
#pragma unroll 8
    for (uint32_t k = lane * 8; k < C; k += 32 * 8) {
      float wv[8];
      load8(wr + k, wv);
#pragma unroll
      for (int i = 0; i < 8; ++i) acc = fmaf(wv[i], pooled[k + i], acc);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0) {
      float v = act_f(acc + a.bias[row], a.act);
      if (a.flags & LF_FINAL)
        static_cast<float*>(a.out)[row] = v;
      else
        static_cast<T*>(a.out)[a.out_co + row] = (T)v;
    }
  }
  mark(5);
  asm volatile("barrier.cluster.wait.aligned;" ::: "memory");
  mark(6);
  instr_exit<INSTR>(ia);
  mark(7);
}

// ---------------------------------------------------------------------------
// Synthetic kernel of the HoL microbenchmark (Fig. 2, P431-445): one block stays
// resident a.kh microseconds (globaltimer) and copies its 8-channel 1x1 input.
// ---------------------------------------------------------------------------
template <typename T, bool INSTR>
__global__ void __launch_bounds__(128) k_spin(const __grid_constant__ LayerArgs a,
                                              const __grid_constant__ InstrArgs ia) {
  kernel_begin<INSTR>(ia);
  if (threadIdx.x == 0) {
    float v[8];
    load8(static_cast<const T*>(a.in) + a.in_co, v);
    const uint64_t t0 = globaltimer(), dur = (uint64_t)a.kh * 1000u;
    while (globaltimer() - t0 < dur) __nanosleep(200);
    store8(static_cast<T*>(a.out) + a.out_co, v);
  }
  instr_exit<INSTR>(ia);
}

// ---------------------------------------------------------------------------
// Empty instrumented kernel for the notification microbenchmark (K5, Fig. 15).
// ---------------------------------------------------------------------------
template <bool INSTR>
__global__ void k_empty(const __grid_constant__ LayerArgs a, const __grid_constant__ InstrArgs ia) {
  kernel_begin<INSTR>(ia);
  instr_exit<INSTR>(ia);
}

// ---------------------------------------------------------------------------
// Gate: holds a stream until the host sets *flag (mapped host memory), so that the
// kernels queued behind it run back to back and CUDA events time the device only.
// ---------------------------------------------------------------------------
__global__ void k_gate(const volatile uint32_t* flag) {
  while (*flag == 0) __nanosleep(1000);
}

KernelFn gate_kernel() { return (KernelFn)k_gate; }

// globaltimer -> host clock calibration (SURVEY.md §8(c) C3 "Clocks"): ping-pong with the
// host through mapped memory.  For i < n: wait until the host raises flag to i + 1, read
// %globaltimer, publish it in out[i].  Then out[n] = the smallest positive step between
// consecutive %globaltimer reads (the timer's resolution, measured, not assumed).
__global__ void k_clock_probe(const volatile uint32_t* flag, volatile unsigned long long* out, uint32_t n) {
  for (uint32_t i = 0; i < n; ++i) {
    while (*flag != i + 1) {
    }
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    out[i] = t;
    __threadfence_system();
  }
  unsigned long long prev, best = ~0ull;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(prev));
  for (int k = 0; k < 20000; ++k) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t != prev) {
      if (t - prev < best) best = t - prev;
      prev = t;
    }
  }
  out[n] = best;
  __threadfence_system();
}

KernelFn clock_kernel() { return (KernelFn)k_clock_probe; }

// ---------------------------------------------------------------------------
// Notification proxy: one persistent warp forwards records from the device-memory
// ring (where the instrumented kernels write them: an L2 store, no PCIe write on the
// kernels' exit path) to the pinned host ring the dispatcher polls.  Lane i checks
// slot head+i; the valid prefix of the window is copied with one 16-byte store per
// lane and the device slots are cleared.  Order and lap tags are preserved, so the
// host sees exactly the records it would see with direct writes.
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(32, 1) k_notify_proxy(const Rec* dev_ring, Rec* host_ring, uint32_t mask,
                                                        uint32_t log2cap, volatile uint32_t* state) {
  // state (pinned, mapped): [0] stop request, [16] heartbeat, [32] exited flag,
  // [48] ring index to resume from.  The warp leaves on its own after ~20 ms without
  // records (so device-wide synchronisation elsewhere in the process can never wait
  // on it forever); the dispatcher relaunches it when it has records outstanding.
  const uint32_t lane = threadIdx.x;
  uint32_t head = state[48];
  uint32_t idle = 0;
  for (;;) {
    const uint32_t idx = head + lane;
    const Rec* src = dev_ring + (idx & mask);
    uint64_t w0, w1;
    asm volatile("ld.volatile.global.v2.u64 {%0, %1}, [%2];" : "=l"(w0), "=l"(w1) : "l"(src));
    const uint32_t tag = rec_tag(idx >> log2cap);
    const bool valid = (w0 & 0xff) != REC_INVALID && ((w0 >> 24) & 0xff) == tag && (w1 >> 56) == tag;
    const uint32_t bal = __ballot_sync(0xffffffffu, valid);
    const uint32_t n = (bal == 0xffffffffu) ? 32u : (uint32_t)(__ffs(~bal) - 1);   // valid prefix
    if (lane < n) {
      Rec* dst = host_ring + (idx & mask);
      asm volatile("st.global.v2.u64 [%0], {%1, %2};" ::"l"(dst), "l"(w0), "l"(w1) : "memory");
      asm volatile("st.global.v2.u64 [%0], {%1, %2};" ::"l"(src), "l"(0ull), "l"(0ull) : "memory");
    }
    head += n;
    if (n == 0) {
      ++idle;
      if ((idle & 255) == 0) {
        if (state[0] || idle > (1u << 16)) break;
        if (lane == 0) state[16] = head;
      }
      __nanosleep(64);
    } else {
      idle = 0;
    }
  }
  if (lane == 0) {
    state[48] = head;
    __threadfence_system();
    state[32] = 1;
  }
}

KernelFn proxy_kernel() { return (KernelFn)k_notify_proxy; }

// ---------------------------------------------------------------------------
// Counter mirror (counter-mode notification): one resident warp copies
// the NCTR_M {start, end} launch counters (NCTR_SUB tables of 2 KiB in device memory,
// summed) to one 2 KiB table in pinned host memory whenever they change.  Lane i owns
// 16-byte chunks i, i+32, i+64, i+96 of every table (two slots each).  A changed sum is
// published after the acquire loads of its parts, so the host sees a block's outputs
// no later than the count that covers the block.  The warp leaves
// after ~35 ms without changes; the dispatcher relaunches it while launches are in
// flight (the counters are the state, so nothing is lost across a relaunch).
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(32, 1) k_notify_mirror(const uint4* ctrs, uint4* host, volatile uint32_t* state) {
  const uint32_t pace = state[8];   // diagnosis (PAELLA_MIRROR_PACE_NS): extra pause per scan
  const uint32_t lane = threadIdx.x;
  // the NCTR_SUB device tables are summed here, so the host reads ONE table of NCTR_M
  // {start, end} pairs (a quarter of the cache lines its drain loop misses on)
  constexpr uint32_t NT = NCTR_M * 2 / 4 / 32;   // 16-byte chunks per lane of one table
  constexpr uint32_t NQ = NCTR_SUB * NT;          // ... of all tables
  uint4 prev[NT];
#pragma unroll
  for (uint32_t i = 0; i < NT; ++i) prev[i] = make_uint4(~0u, ~0u, ~0u, ~0u);   // publish everything once
  uint32_t idle = 0;
  for (;;) {
    uint4 raw[NQ];
#pragma unroll
    for (uint32_t i = 0; i < NQ; ++i)
      asm volatile("ld.acquire.gpu.global.v4.u32 {%0, %1, %2, %3}, [%4];"
                   : "=r"(raw[i].x), "=r"(raw[i].y), "=r"(raw[i].z), "=r"(raw[i].w)
                   : "l"(ctrs + lane + 32 * i));
    uint4 cur[NT];
    bool ch = false;
#pragma unroll
    for (uint32_t q = 0; q < NT; ++q) {
      cur[q] = raw[q];
#pragma unroll
      for (uint32_t t = 1; t < NCTR_SUB; ++t) {
        cur[q].x += raw[t * NT + q].x;
        cur[q].y += raw[t * NT + q].y;
        cur[q].z += raw[t * NT + q].z;
        cur[q].w += raw[t * NT + q].w;
      }
      ch |= cur[q].x != prev[q].x || cur[q].y != prev[q].y || cur[q].z != prev[q].z || cur[q].w != prev[q].w;
    }
    if (__any_sync(0xffffffffu, ch)) {
      // A block's release reduction made its outputs visible (at system scope for a
      // job's last kernel) before its count could be loaded with acquire; PTX gives no
      // ordering from the load->store data dependency, so one system-scope fence per
      // batch of changed chunks orders those outputs before the relaxed stores that
      // publish the counts to the host (cumulativity of fence.acq_rel.sys)
      asm volatile("fence.acq_rel.sys;" ::: "memory");
#pragma unroll
      for (uint32_t i = 0; i < NT; ++i) {
        if (cur[i].x != prev[i].x || cur[i].y != prev[i].y || cur[i].z != prev[i].z || cur[i].w != prev[i].w) {
          asm volatile("st.relaxed.sys.global.v4.u32 [%0], {%1, %2, %3, %4};" ::"l"(host + lane + 32 * i),
                       "r"(cur[i].x), "r"(cur[i].y), "r"(cur[i].z), "r"(cur[i].w)
                       : "memory");
          prev[i] = cur[i];
        }
      }
      idle = 0;
    } else {
      ++idle;
      if ((idle & 255) == 0) {
        if (state[0] || idle > (1u << 16)) break;
        if (lane == 0) state[16] = idle;
      }
      __nanosleep(64);
    }
    if (pace) __nanosleep(pace);
  }
  if (lane == 0) {
    __threadfence_system();
    state[32] = 1;
  }
}

KernelFn mirror_kernel() { return (KernelFn)k_notify_mirror; }

// ---------------------------------------------------------------------------
// kernel table
// ---------------------------------------------------------------------------
template <typename T, bool I>
static void fill(KernelFn (&t)[KIND_COUNT]) {
  t[KIND_INGEST] = (KernelFn)k_ingest<T, I>;
  t[KIND_CONV_SIMT] = (KernelFn)k_conv_simt<T, I>;
  t[KIND_DWCONV] = (KernelFn)k_dwconv<T, I>;
  t[KIND_MAXPOOL] = (KernelFn)k_pool<T, I, true>;
  t[KIND_AVGPOOL] = (KernelFn)k_pool<T, I, false>;
  t[KIND_GAP] = (KernelFn)k_gap<T, I>;
  t[KIND_FC] = (KernelFn)k_fc<T, I>;
  t[KIND_EMPTY] = (KernelFn)k_empty<I>;
  t[KIND_GAPFC] = (KernelFn)k_gapfc<T, I>;
  t[KIND_SPIN] = (KernelFn)k_spin<T, I>;
}

void simt_kernel_table(KernelFn (&bf16_instr)[KIND_COUNT], KernelFn (&bf16_plain)[KIND_COUNT],
                       KernelFn (&f32_instr)[KIND_COUNT], KernelFn (&f32_plain)[KIND_COUNT]) {
  fill<__nv_bfloat16, true>(bf16_instr);
  fill<__nv_bfloat16, false>(bf16_plain);
  fill<float, true>(f32_instr);
  fill<float, false>(f32_plain);
}

}  // namespace paella
