// Probe 2: front-end stream memop costs and wake-up latency.
//  a) cost of n back-to-back cuStreamWriteValue32 in one stream (events around), with and without
//     CU_STREAM_WRITE_VALUE_NO_MEMORY_BARRIER
//  b) wake-up latency of cuStreamWaitValue32 when the value is written by a running kernel
//     (device %globaltimer: writer's store -> first CTA of the gated kernel)
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#define CK(x) do { cudaError_t e = (x); if (e) { printf("CUDA %s line %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)
__device__ __forceinline__ uint64_t gt() { uint64_t r; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(r)); return r; }
__global__ void k_writer(uint32_t* flag, uint64_t* t, uint64_t spin_ns) {
  uint64_t t0 = gt(); while (gt() - t0 < spin_ns) {}
  t[0] = gt(); atomicExch(flag, 1u);
}
__global__ void k_stamp(uint64_t* t) { if (threadIdx.x == 0 && blockIdx.x == 0) t[1] = gt(); }
__global__ void k_empty() {}
typedef CUresult (*PFN)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
int main() {
  PFN wv = nullptr, wt = nullptr; cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuStreamWriteValue32", (void**)&wv, cudaEnableDefault, &q));
  CK(cudaGetDriverEntryPoint("cuStreamWaitValue32", (void**)&wt, cudaEnableDefault, &q));
  cudaStream_t s1, s2; CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking)); CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
  uint32_t* d; CK(cudaMalloc(&d, 64 * 4)); uint64_t* t; CK(cudaMalloc(&t, 16));
  cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  for (int flags : {0, 1}) {
    for (int n : {0, 1, 6, 24}) {
      std::vector<float> v;
      for (int r = 0; r < 50; r++) {
        k_empty<<<1, 32, 0, s1>>>();
        CK(cudaEventRecord(e0, s1));
        for (int i = 0; i < n; i++) wv((CUstream)s1, (CUdeviceptr)(d + i % 64), 0, flags);
        k_empty<<<1, 32, 0, s1>>>();
        CK(cudaEventRecord(e1, s1)); CK(cudaEventSynchronize(e1));
        float ms; CK(cudaEventElapsedTime(&ms, e0, e1)); v.push_back(ms * 1000);
      }
      std::sort(v.begin(), v.end());
      printf("{\"probe\":\"memop_chain\",\"no_barrier\":%d,\"n\":%d,\"us_p50\":%.2f,\"min\":%.2f}\n", flags, n, v[25], v[0]);
    }
  }
  for (uint64_t spin : {20000ull, 200000ull}) {
    std::vector<double> lat;
    for (int r = 0; r < 30; r++) {
      CK(cudaMemset(d, 0, 4)); CK(cudaDeviceSynchronize());
      wt((CUstream)s2, (CUdeviceptr)d, 1, CU_STREAM_WAIT_VALUE_GEQ);
      k_stamp<<<1, 32, 0, s2>>>(t);
      k_writer<<<1, 1, 0, s1>>>(d, t, spin);
      CK(cudaDeviceSynchronize());
      uint64_t h[2]; CK(cudaMemcpy(h, t, 16, cudaMemcpyDeviceToHost));
      lat.push_back((double)(h[1] - h[0]) / 1000.0);
    }
    std::sort(lat.begin(), lat.end());
    printf("{\"probe\":\"wait_value_wakeup\",\"writer_spin_us\":%llu,\"us_p50\":%.2f,\"min\":%.2f,\"max\":%.2f}\n",
           (unsigned long long)spin / 1000, lat[15], lat[0], lat.back());
  }
  // launch gating by a plain event on another stream's kernel completion (for comparison)
  {
    std::vector<double> lat;
    for (int r = 0; r < 30; r++) {
      cudaEvent_t ev; CK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
      k_writer<<<1, 1, 0, s1>>>(d, t, 20000);
      CK(cudaEventRecord(ev, s1)); CK(cudaStreamWaitEvent(s2, ev, 0));
      k_stamp<<<1, 32, 0, s2>>>(t);
      CK(cudaDeviceSynchronize());
      uint64_t h[2]; CK(cudaMemcpy(h, t, 16, cudaMemcpyDeviceToHost));
      lat.push_back((double)(h[1] - h[0]) / 1000.0);
      cudaEventDestroy(ev);
    }
    std::sort(lat.begin(), lat.end());
    printf("{\"probe\":\"event_gate\",\"us_p50\":%.2f,\"min\":%.2f,\"max\":%.2f}\n", lat[15], lat[0], lat.back());
  }
  return 0;
}
