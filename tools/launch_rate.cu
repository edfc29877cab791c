// Diagnosis: host-side kernel launch throughput on one context, the bound on how many
// kernels per second a software dispatcher can issue (Paella issues every kernel of every
// job itself, ~73 per C-3 request).  T threads each own S streams and launch an empty
// kernel carrying a Paella-sized parameter block (~360 B: LayerArgs + InstrArgs + a
// 128 B tensor map) as fast as they can; aggregate launches/s per API:
//   0 cudaLaunchKernel                     (no attributes)
//   1 cudaLaunchKernelExC + PDL attribute  (what the dispatcher's launchers call)
//   2 cuLaunchKernelEx (driver API) + PDL
//   3 cudaLaunchKernelExC + PDL + cluster (1,1,16), grid 64
//   4 cuLaunchKernelEx + PDL + cluster (1,1,16), grid 64
//   5 cudaLaunchKernelExC + PDL, 64 B parameter block
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/lr tools/launch_rate.cu -lcuda -lpthread
#include <cuda.h>
#include <cuda_runtime.h>

#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <thread>
#include <vector>

struct Params {
  unsigned char b[352];
};
struct Small {
  unsigned char b[64];
};

__global__ void empty_k(const __grid_constant__ Params p) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  if (p.b[0] == 255 && threadIdx.x == 9999) printf("x");
}
__global__ void empty_small(const __grid_constant__ Small p) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  if (p.b[0] == 255 && threadIdx.x == 9999) printf("x");
}

static double run(int mode, int T, int S, int per_thread) {
  std::vector<std::vector<cudaStream_t>> st(T);
  for (int t = 0; t < T; ++t)
    for (int s = 0; s < S; ++s) {
      cudaStream_t x;
      cudaStreamCreateWithFlags(&x, cudaStreamNonBlocking);
      st[t].push_back(x);
    }
  CUfunction cf = nullptr;
  cudaGetFuncBySymbol(&cf, (const void*)empty_k);
  std::atomic<int> go{0};
  std::vector<std::thread> th;
  std::atomic<long> done{0};
  auto body = [&](int t) {
    cudaSetDevice(0);
    Params p{};
    Small ps{};
    void* args[1] = {&p};
    void* args_s[1] = {&ps};
    while (!go.load()) {
    }
    for (int i = 0; i < per_thread; ++i) {
      cudaStream_t s = st[t][i % S];
      const bool cl = mode >= 3;
      const unsigned gz = cl ? 64 : 1;
      if (mode == 0) {
        cudaLaunchKernel((const void*)empty_k, dim3(1, 1, gz), dim3(128), args, 0, s);
      } else if (mode == 5) {   // PDL, 64 B parameter block
        cudaLaunchConfig_t cfg{};
        cfg.gridDim = dim3(1, 1, 1);
        cfg.blockDim = dim3(128);
        cfg.stream = s;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        at[0].val.programmaticStreamSerializationAllowed = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        cudaLaunchKernelExC(&cfg, (const void*)empty_small, args_s);
      } else if (mode == 1 || mode == 3) {
        cudaLaunchConfig_t cfg{};
        cfg.gridDim = dim3(1, 1, gz);
        cfg.blockDim = dim3(128);
        cfg.stream = s;
        cudaLaunchAttribute at[2];
        int n = 0;
        at[n].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        at[n].val.programmaticStreamSerializationAllowed = 1;
        ++n;
        if (cl) {
          at[n].id = cudaLaunchAttributeClusterDimension;
          at[n].val.clusterDim.x = 1;
          at[n].val.clusterDim.y = 1;
          at[n].val.clusterDim.z = 16;
          ++n;
        }
        cfg.attrs = at;
        cfg.numAttrs = n;
        cudaLaunchKernelExC(&cfg, (const void*)empty_k, args);
      } else {
        CUlaunchConfig cfg{};
        cfg.gridDimX = 1;
        cfg.gridDimY = 1;
        cfg.gridDimZ = gz;
        cfg.blockDimX = 128;
        cfg.blockDimY = 1;
        cfg.blockDimZ = 1;
        cfg.hStream = (CUstream)s;
        CUlaunchAttribute at[2];
        int n = 0;
        at[n].id = CU_LAUNCH_ATTRIBUTE_PROGRAMMATIC_STREAM_SERIALIZATION;
        at[n].value.programmaticStreamSerializationAllowed = 1;
        ++n;
        if (cl) {
          at[n].id = CU_LAUNCH_ATTRIBUTE_CLUSTER_DIMENSION;
          at[n].value.clusterDim.x = 1;
          at[n].value.clusterDim.y = 1;
          at[n].value.clusterDim.z = 16;
          ++n;
        }
        cfg.attrs = at;
        cfg.numAttrs = n;
        cuLaunchKernelEx(&cfg, cf, args, nullptr);
      }
    }
    done.fetch_add(per_thread);
  };
  for (int t = 0; t < T; ++t) th.emplace_back(body, t);
  auto t0 = std::chrono::steady_clock::now();
  go.store(1);
  for (auto& x : th) x.join();
  auto t1 = std::chrono::steady_clock::now();
  cudaDeviceSynchronize();
  const double s = std::chrono::duration<double>(t1 - t0).count();
  for (auto& v : st)
    for (auto x : v) cudaStreamDestroy(x);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) fprintf(stderr, "error %s\n", cudaGetErrorString(e));
  return done.load() / s;
}

int main(int argc, char** argv) {
  const int per = argc > 1 ? atoi(argv[1]) : 40000;
  cudaSetDevice(0);
  cudaFree(0);
  run(1, 1, 8, 2000);   // warm-up
  printf("mode threads streams_per_thread launches_per_s us_per_launch_per_thread\n");
  for (int mode : {1, 5, 0, 2})
    for (int T : {1, 2, 4, 8}) {
      const double r = run(mode, T, 8, per);
      printf("%d %d %d %.0f %.3f\n", mode, T, 8, r, 1e6 * T / r);
      fflush(stdout);
    }
  return 0;
}
