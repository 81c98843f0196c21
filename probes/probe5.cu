// Probe 5: launch-side costs of a wrapped grid outside its workers' span. A grid of
// W CTAs spins ~2 us (%globaltimer) and exits; timed with CUDA events behind a gate kernel:
//   small      : 16-B kernel parameters
//   params256  : 256-B kernel parameters (the wrapper's Args + WorkerParams are ~200 B)
//   event_after: small + a timing-disabled cudaEventRecord right after the grid (the runtime's
//                completion event)
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#define CK(x) do { cudaError_t e = (x); if (e) { printf("CUDA %s line %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__global__ void k_gate(uint64_t ns) {
  uint64_t t0; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  while (true) { uint64_t t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); if (t - t0 > ns) break; __nanosleep(1000); }
}
__device__ __forceinline__ void spin(uint64_t ns) {
  uint64_t t0; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  while (true) { uint64_t t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); if (t - t0 > ns) break; }
}
struct Big { uint64_t w[32]; };
__global__ void k_small(uint64_t ns, uint32_t* out) { spin(ns); if (threadIdx.x == 0 && ns == 1) out[blockIdx.x] = 1; }
__global__ void k_big(const __grid_constant__ Big b, uint32_t* out) { spin(b.w[0]); if (threadIdx.x == 0 && b.w[31] == 7) out[blockIdx.x] = 1; }

int main() {
  int nsm; CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  uint32_t* out; CK(cudaMalloc(&out, 1 << 20));
  cudaStream_t s; CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  cudaEvent_t e0, e1, ex; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  CK(cudaEventCreateWithFlags(&ex, cudaEventDisableTiming));
  const char* names[] = {"small", "params256", "event_after"};
  Big b{}; b.w[0] = 2000;
  for (uint32_t W : {(uint32_t)nsm * 4, (uint32_t)nsm * 8}) {
    for (int mode = 0; mode < 3; ++mode) {
      std::vector<float> v;
      for (int r = 0; r < 100; ++r) {
        k_gate<<<1, 32, 0, s>>>(100000 + 37 * (r % 29));
        CK(cudaEventRecord(e0, s));
        if (mode == 1) k_big<<<W, 256, 0, s>>>(b, out);
        else k_small<<<W, 256, 0, s>>>(2000, out);
        if (mode == 2) CK(cudaEventRecord(ex, s));
        CK(cudaEventRecord(e1, s)); CK(cudaEventSynchronize(e1));
        float ms; CK(cudaEventElapsedTime(&ms, e0, e1)); v.push_back(ms * 1000.f);
      }
      std::sort(v.begin(), v.end());
      double m = 0; for (size_t i = 10; i < 90; ++i) m += v[i]; m /= 80;
      printf("{\"probe\":\"launch_side\",\"case\":\"%s\",\"ctas\":%u,\"us_mean80\":%.3f,\"min\":%.3f}\n",
             names[mode], W, m, v[0]);
    }
  }
  return 0;
}
