// Probe 3: what a kernel boundary costs on the GPU (SURVEY §8(d) latency floors; DESIGN §6 wrapper
// overhead). Every case is timed with CUDA events behind a __nanosleep gate kernel (so that host
// submission latency is hidden), single launch and 10 back-to-back launches.
//   empty      : W CTAs that return immediately
//   dev_last   : + the last CTA (64-bit atomic counter) writes 8 B to device memory
//   sys_last   : + the last CTA writes 8 B to mapped pinned HOST memory (st.relaxed.sys)
//   sys_entry  : + CTA 0 also writes 4 B to host memory at entry (the wrapper's "started" hint)
//   evlog      : + every CTA writes a 32-B record and does one 64-bit atomic (the wrapper's exit)
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

template <int kMode>
__global__ void k_case(unsigned long long* ctr, uint64_t* dev, uint64_t* host, uint4* ev, uint32_t W) {
  if (threadIdx.x != 0) return;
  if (kMode >= 3 && blockIdx.x == 0)
    asm volatile("st.relaxed.sys.global.u32 [%0], %1;" :: "l"(host + 1), "r"(1u) : "memory");
  if (kMode == 0) return;
  if (kMode >= 4) ev[blockIdx.x * 2] = make_uint4(blockIdx.x, 1, 2, 3);
  const unsigned long long old = atomicAdd(ctr, 1ull);
  if ((uint32_t)old + 1 == W) {
    *ctr = 0;
    if (kMode == 1) *dev = old;
    else asm volatile("st.relaxed.sys.global.u64 [%0], %1;" :: "l"(host), "l"((uint64_t)old) : "memory");
  }
}

int main() {
  int nsm; CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  unsigned long long* ctr; uint64_t* dev; uint4* ev; uint64_t* host; uint64_t* dhost;
  CK(cudaMalloc(&ctr, 8)); CK(cudaMemset(ctr, 0, 8)); CK(cudaMalloc(&dev, 8)); CK(cudaMalloc(&ev, 1 << 20));
  CK(cudaHostAlloc(&host, 64, cudaHostAllocMapped)); CK(cudaHostGetDevicePointer(&dhost, host, 0));
  cudaStream_t s; CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  const char* names[] = {"empty", "dev_last", "sys_last", "sys_entry", "evlog"};
  for (uint32_t W : {(uint32_t)nsm * 8, (uint32_t)nsm * 4}) {
    for (int mode = 0; mode < 5; ++mode) {
      for (int reps : {1, 10}) {
        std::vector<float> v;
        for (int r = 0; r < 40; ++r) {
          k_gate<<<1, 32, 0, s>>>(200000);
          CK(cudaEventRecord(e0, s));
          for (int i = 0; i < reps; ++i) {
            switch (mode) {
              case 0: k_case<0><<<W, 256, 0, s>>>(ctr, dev, dhost, ev, W); break;
              case 1: k_case<1><<<W, 256, 0, s>>>(ctr, dev, dhost, ev, W); break;
              case 2: k_case<2><<<W, 256, 0, s>>>(ctr, dev, dhost, ev, W); break;
              case 3: k_case<3><<<W, 256, 0, s>>>(ctr, dev, dhost, ev, W); break;
              default: k_case<4><<<W, 256, 0, s>>>(ctr, dev, dhost, ev, W); break;
            }
          }
          CK(cudaEventRecord(e1, s)); CK(cudaEventSynchronize(e1));
          float ms; CK(cudaEventElapsedTime(&ms, e0, e1)); v.push_back(ms * 1000.f / reps);
        }
        std::sort(v.begin(), v.end());
        printf("{\"probe\":\"kernel_boundary\",\"case\":\"%s\",\"ctas\":%u,\"b2b\":%d,\"us_per_launch_p50\":%.2f,\"min\":%.2f}\n",
               names[mode], W, reps, v[v.size() / 2], v[0]);
      }
    }
  }
  return 0;
}
