// Diagnosis: per-launch time of back-to-back dependent kernels on one stream as a
// function of the kernel's own duration (a globaltimer spin), plain launches vs
// programmatic dependent launch (PDL) vs a CUDA graph.  Tells whether kernel
// boundaries cost a fixed quantum on this GPU.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/lq tools/launch_quantum.cu
#include <chrono>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned long long gt() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
__global__ void spin(unsigned ns, int pdl) {
  if (pdl) asm volatile("griddepcontrol.wait;" ::: "memory");
  unsigned long long t0 = gt();
  while (gt() - t0 < ns) {
  }
  if (pdl) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
__global__ void gate(volatile int* g) {
  while (*g == 0) {
  }
}

int main() {
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  int* gh;
  cudaHostAlloc(&gh, 4, cudaHostAllocMapped);
  int* gd;
  cudaHostGetDevicePointer(&gd, gh, 0);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int R = 200;
  printf("spin_ns grid plain_us pdl_us graph_us\n");
  for (int grid : {1, 16}) {
    for (unsigned ns = 0; ns <= 8000; ns += 500) {
      float res[3];
      for (int mode = 0; mode < 3; ++mode) {
        cudaGraphExec_t ge = nullptr;
        if (mode == 2) {
          cudaGraph_t g;
          cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal);
          for (int r = 0; r < R; ++r) spin<<<grid, 128, 0, s>>>(ns, 0);
          cudaStreamEndCapture(s, &g);
          cudaGraphInstantiate(&ge, g, 0);
          cudaGraphDestroy(g);
        }
        *gh = 0;
        gate<<<1, 1, 0, s>>>(gd);
        cudaEventRecord(e0, s);
        if (mode == 0) {
          for (int r = 0; r < R; ++r) spin<<<grid, 128, 0, s>>>(ns, 0);
        } else if (mode == 1) {
          cudaLaunchConfig_t cfg = {};
          cfg.gridDim = grid;
          cfg.blockDim = 128;
          cfg.stream = s;
          cudaLaunchAttribute at[1];
          at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
          at[0].val.programmaticStreamSerializationAllowed = 1;
          cfg.attrs = at;
          cfg.numAttrs = 1;
          for (int r = 0; r < R; ++r) cudaLaunchKernelEx(&cfg, spin, ns, 1);
        } else {
          cudaGraphLaunch(ge, s);
        }
        cudaEventRecord(e1, s);
        __sync_synchronize();
        *(volatile int*)gh = 1;
        cudaStreamSynchronize(s);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        res[mode] = ms * 1000.f / R;
        if (ge) cudaGraphExecDestroy(ge);
      }
      printf("%u %d %.3f %.3f %.3f\n", ns, grid, res[0], res[1], res[2]);
    }
  }

  // front-end throughput: S streams, each R back-to-back kernels (spin ns), all gated
  printf("streams spin_ns grid kernels_per_s plain | pdl   host_us_per_launch plain | pdl\n");
  cudaStream_t ss[64];
  for (int i = 0; i < 64; ++i) cudaStreamCreateWithFlags(&ss[i], cudaStreamNonBlocking);
  for (int S : {1, 4, 16, 32, 64}) {
    for (unsigned ns : {0u, 2000u, 5000u}) {
      double kps[2], hus[2];
      for (int mode = 0; mode < 2; ++mode) {
        const int RR = 100;
        *gh = 0;
        for (int i = 0; i < S; ++i) gate<<<1, 1, 0, ss[i]>>>(gd);
        cudaEventRecord(e0, ss[0]);
        auto t0 = std::chrono::steady_clock::now();
        for (int r = 0; r < RR; ++r)
          for (int i = 0; i < S; ++i) {
            if (mode == 0) {
              spin<<<8, 128, 0, ss[i]>>>(ns, 0);
            } else {
              cudaLaunchConfig_t cfg = {};
              cfg.gridDim = 8;
              cfg.blockDim = 128;
              cfg.stream = ss[i];
              cudaLaunchAttribute at[1];
              at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
              at[0].val.programmaticStreamSerializationAllowed = 1;
              cfg.attrs = at;
              cfg.numAttrs = 1;
              cudaLaunchKernelEx(&cfg, spin, ns, 1);
            }
          }
        auto t1 = std::chrono::steady_clock::now();
        hus[mode] = std::chrono::duration<double, std::micro>(t1 - t0).count() / (RR * S);
        for (int i = 1; i < S; ++i) {
          cudaEvent_t ev;
          cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
          cudaEventRecord(ev, ss[i]);
          cudaStreamWaitEvent(ss[0], ev, 0);
          cudaEventDestroy(ev);
        }
        cudaEventRecord(e1, ss[0]);
        __sync_synchronize();
        *(volatile int*)gh = 1;
        cudaDeviceSynchronize();
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        kps[mode] = RR * S / (ms * 1e-3);
      }
      printf("%d %u 8 %.0f | %.0f   %.2f | %.2f\n", S, ns, kps[0], kps[1], hus[0], hus[1]);
    }
  }
  cudaStream_t s2;
  cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
  printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
