// Diagnosis: how fast can ONE SM fill its shared memory from L2?  The batch-1 conv's
// k-block loop moves ~24 KB per k-block into shared memory (16 KB weights by TMA + 8 KB
// gathered activations) and runs at ~260 ns per k-block whatever the ring depth
// (profiles/r2/diag/kblock): if the per-SM L2 -> SMEM fill rate is ~90-100 GB/s, that
// is the bound.  An L2-resident buffer (4 MB) is streamed into a shared-memory ring by
//   mode 0: one thread issuing 1-D bulk copies (cp.async.bulk, mbarrier complete_tx),
//           CH bytes each, STG in flight (the weight path's mechanism);
//   mode 1: 128 threads issuing 16 B cp.async (LDGSTS), one commit group per chunk,
//           STG groups in flight (the activation gather's mechanism);
// for grids of 1, 16, 74, 148 and 296 CTAs (CTA i reads its own rotating offsets).
// Per CTA globaltimer span -> GB/s per CTA, per SM and aggregate.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/l2bw tools/l2_fill_bw.cu
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <vector>

constexpr int STG = 8;

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

__global__ void k_bulk(const char* src, uint32_t buf_bytes, uint32_t ch, int iters, uint64_t* span) {
  extern __shared__ __align__(1024) char sm[];
  __shared__ __align__(8) uint64_t bar[STG];
  if (threadIdx.x == 0) {
    for (int s = 0; s < STG; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[s])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x != 0) return;
  const uint64_t t0 = gtimer();
  const uint32_t nchunks = buf_bytes / ch;
  for (int i = 0; i < iters; ++i) {
    const int s = i % STG;
    if (i >= STG) {
      const uint32_t par = ((i / STG) - 1) & 1;
      asm volatile(
          "{\n\t.reg .pred p;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n}" ::"r"(
              su32(&bar[s])),
          "r"(par)
          : "memory");
    }
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[s])), "r"(ch) : "memory");
    const char* g = src + (size_t)((blockIdx.x * 7 + i) % nchunks) * ch;
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     su32(sm + s * ch)),
                 "l"(g), "r"(ch), "r"(su32(&bar[s]))
                 : "memory");
  }
  for (int i = iters; i < iters + STG; ++i) {
    const int s = i % STG;
    const uint32_t par = ((i / STG) - 1) & 1;
    if (i - STG >= 0)
      asm volatile(
          "{\n\t.reg .pred p;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n}" ::"r"(
              su32(&bar[s])),
          "r"(par)
          : "memory");
  }
  span[blockIdx.x] = gtimer() - t0;
}

__global__ void k_ldgsts(const char* src, uint32_t buf_bytes, uint32_t ch, int iters, uint64_t* span) {
  extern __shared__ __align__(1024) char sm[];
  __syncthreads();
  const uint64_t t0 = gtimer();
  const uint32_t nchunks = buf_bytes / ch;
  for (int i = 0; i < iters; ++i) {
    const int s = i % STG;
    const char* g = src + (size_t)((blockIdx.x * 7 + i) % nchunks) * ch;
    for (uint32_t o = threadIdx.x * 16; o < ch; o += blockDim.x * 16)
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(su32(sm + s * ch + o)), "l"(g + o) : "memory");
    asm volatile("cp.async.commit_group;" ::: "memory");
    asm volatile("cp.async.wait_group %0;" ::"n"(STG - 1) : "memory");
  }
  asm volatile("cp.async.wait_group 0;" ::: "memory");
  __syncthreads();
  if (threadIdx.x == 0) span[blockIdx.x] = gtimer() - t0;
}

int main() {
  const uint32_t buf = 4u << 20;
  char* src;
  uint64_t* span;
  cudaMalloc(&src, buf);
  cudaMemset(src, 1, buf);
  cudaMalloc(&span, 1024 * sizeof(uint64_t));
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  printf("mode chunk_B grid ctas_per_sm median_span_us GBps_per_cta GBps_per_sm aggregate_GBps\n");
  for (int mode : {0, 1})
    for (uint32_t ch : {8192u, 16384u})
      for (int grid : {1, 16, 74, sms, 2 * sms}) {
        const int iters = 2000;
        const size_t smem = (size_t)STG * ch;
        auto kern = mode == 0 ? k_bulk : k_ldgsts;
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        int occ = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, 128, smem);
        if (grid > occ * sms) continue;   // one wave only
        for (int rep = 0; rep < 3; ++rep) kern<<<grid, 128, smem>>>(src, buf, ch, iters, span);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) {
          printf("error %s\n", cudaGetErrorString(e));
          return 1;
        }
        std::vector<uint64_t> h(grid);
        cudaMemcpy(h.data(), span, grid * sizeof(uint64_t), cudaMemcpyDeviceToHost);
        std::sort(h.begin(), h.end());
        const double med = (double)h[grid / 2], mx = (double)h.back();
        const double bytes = (double)iters * ch;
        const int per_sm = grid > sms ? 2 : 1;
        printf("%d %u %d %d %.1f %.1f %.1f %.0f\n", mode, ch, grid, per_sm, med / 1e3, bytes / med,
               per_sm * bytes / med, grid * bytes / mx);
        fflush(stdout);
      }
  return 0;
}
