// Probe 4: which part of the wrapper's exit accounting costs time at a kernel boundary (DESIGN §7
// "wrapper overhead of short kernels"). Same harness as probe3 (gate kernel, CUDA events, single
// launch and 10 back to back). Every CTA's thread 0 does, by case:
//   empty        : nothing
//   red64        : one fire-and-forget 64-bit red.add to one address (no return value)
//   red64_sm     : one red.add to a per-SM line (148 addresses, one 128-B line each)
//   atom64       : one 64-bit atom.add with return (result consumed), nothing else
//   atom64_last  : + the last CTA stores 8 B to device memory (probe3 dev_last)
//   atom64_chain : + the last CTA loads two words (one round trip) and stores 24 B to mapped host
//                  memory (the round-1 wrapper's exit chain)
//   atom64_sys   : + the last CTA stores 8 B to mapped host memory without the loads
//   rec32        : every CTA stores a 32-B record (the wrapper's per-worker event log), no atomic
//   fetch_first  : every CTA does one atomic with return at ENTRY (the exhausted task fetch) and
//                  the W-th one stores 8 B to mapped host memory; nothing at exit
//   fetch_rec    : fetch_first + the 32-B record at exit
//   body_only    : a ~0.5 us stand-in body (spin on %globaltimer), nothing else
//   body_exit_atom: the stand-in body, then the round-1 exit (record, atomic; last -> host store)
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
__global__ void k_case(unsigned long long* ctr, uint32_t* words, uint64_t* dev, uint64_t* host, uint32_t W) {
  if (threadIdx.x != 0) return;
  if (kMode == 0) return;
  if (kMode == 7) { reinterpret_cast<uint4*>(dev + 4)[blockIdx.x * 2] = make_uint4(blockIdx.x, 1, 2, 3); return; }
  if (kMode == 8 || kMode == 9) {
    unsigned long long o;
    asm volatile("atom.relaxed.gpu.global.add.u64 %0, [%1], %2;" : "=l"(o) : "l"(ctr), "l"(1ull) : "memory");
    if ((uint32_t)o + 1 == W) {
      asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" :: "l"(ctr), "l"(0ull) : "memory");
      asm volatile("st.relaxed.sys.global.u64 [%0], %1;" :: "l"(host), "l"((uint64_t)o) : "memory");
    }
    // stand-in for the last body: ~0.5 us of work so the exit is not the fetch itself
    uint64_t t0; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    while (true) { uint64_t t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); if (t - t0 > 500) break; }
    if (kMode == 9) reinterpret_cast<uint4*>(dev + 4)[blockIdx.x * 2] = make_uint4(blockIdx.x, 1, 2, 3);
    return;
  }
  if (kMode >= 10) {   // 10: reference for 8/9, the same ~0.5 us stand-in body, nothing else;
                       // 11: the body, then the round-1 exit (record + atomic, last -> host store)
    uint64_t t0; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    while (true) { uint64_t t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); if (t - t0 > 500) break; }
    if (kMode == 10) return;
    reinterpret_cast<uint4*>(dev + 4)[blockIdx.x * 2] = make_uint4(blockIdx.x, 1, 2, 3);
    unsigned long long o;
    asm volatile("atom.relaxed.gpu.global.add.u64 %0, [%1], %2;" : "=l"(o) : "l"(ctr), "l"(1ull) : "memory");
    if ((uint32_t)o + 1 == W) {
      asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" :: "l"(ctr), "l"(0ull) : "memory");
      asm volatile("st.relaxed.sys.global.u64 [%0], %1;" :: "l"(host), "l"((uint64_t)o) : "memory");
    }
    return;
  }
  if (kMode == 1) { asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" :: "l"(ctr), "l"(1ull) : "memory"); return; }
  if (kMode == 2) {
    uint32_t sm; asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
    asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" :: "l"(ctr + 16 * (sm + 1)), "l"(1ull) : "memory");
    return;
  }
  unsigned long long old;
  asm volatile("atom.relaxed.gpu.global.add.u64 %0, [%1], %2;" : "=l"(old) : "l"(ctr), "l"(1ull) : "memory");
  if ((uint32_t)old + 1 != W) return;
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" :: "l"(ctr), "l"(0ull) : "memory");
  if (kMode == 3) return;
  if (kMode == 4) { *dev = old; return; }
  if (kMode == 5) {
    uint32_t a, b;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(a) : "l"(words) : "memory");
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(b) : "l"(words + 32) : "memory");
    asm volatile("st.relaxed.sys.global.u32 [%0], %1;" :: "l"(host + 2), "r"(a) : "memory");
    asm volatile("st.relaxed.sys.global.u64 [%0], %1;" :: "l"(host + 3), "l"((uint64_t)b) : "memory");
    asm volatile("st.relaxed.sys.global.u64 [%0], %1;" :: "l"(host), "l"((uint64_t)old) : "memory");
    return;
  }
  asm volatile("st.relaxed.sys.global.u64 [%0], %1;" :: "l"(host), "l"((uint64_t)old) : "memory");
}

int main() {
  int nsm; CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  unsigned long long* ctr; uint64_t* dev; uint32_t* words; uint64_t* host; uint64_t* dhost;
  CK(cudaMalloc(&ctr, 128 * 160)); CK(cudaMemset(ctr, 0, 128 * 160)); CK(cudaMalloc(&dev, 1 << 20));
  CK(cudaMalloc(&words, 256)); CK(cudaMemset(words, 0, 256));
  CK(cudaHostAlloc(&host, 64, cudaHostAllocMapped)); CK(cudaHostGetDevicePointer(&dhost, host, 0));
  cudaStream_t s; CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  const char* names[] = {"empty", "red64", "red64_sm", "atom64", "atom64_last", "atom64_chain", "atom64_sys", "rec32", "fetch_first", "fetch_rec", "body_only", "body_exit_atom"};
  for (uint32_t W : {(uint32_t)nsm * 8, (uint32_t)nsm * 4}) {
    for (int mode = 0; mode < 12; ++mode) {
      for (int reps : {1, 10}) {
        std::vector<float> v;
        for (int r = 0; r < 60; ++r) {
          CK(cudaMemsetAsync(ctr, 0, 8, s));
          k_gate<<<1, 32, 0, s>>>(200000);
          CK(cudaEventRecord(e0, s));
          for (int i = 0; i < reps; ++i) {
            switch (mode) {
              case 0: k_case<0><<<W, 256, 0, s>>>(ctr, words, dev, dhost, W); break;
              case 1: k_case<1><<<W, 256, 0, s>>>(ctr, words, dev, dhost, W); break;
              case 2: k_case<2><<<W, 256, 0, s>>>(ctr, words, dev, dhost, W); break;
              case 3: k_case<3><<<W, 256, 0, s>>>(ctr, words, dev, dhost, W); break;
              case 4: k_case<4><<<W, 256, 0, s>>>(ctr, words, dev, dhost, W); break;
              case 5: k_case<5><<<W, 256, 0, s>>>(ctr, words, dev, dhost, W); break;
              case 6: k_case<6><<<W, 256, 0, s>>>(ctr, words, dev, dhost, W); break;
              case 7: k_case<7><<<W, 256, 0, s>>>(ctr, words, dev, dhost, W); break;
              case 8: k_case<8><<<W, 256, 0, s>>>(ctr, words, dev, dhost, W); break;
              case 9: k_case<9><<<W, 256, 0, s>>>(ctr, words, dev, dhost, W); break;
              case 10: k_case<10><<<W, 256, 0, s>>>(ctr, words, dev, dhost, W); break;
              default: k_case<11><<<W, 256, 0, s>>>(ctr, words, dev, dhost, W); break;
            }
          }
          CK(cudaEventRecord(e1, s)); CK(cudaEventSynchronize(e1));
          float ms; CK(cudaEventElapsedTime(&ms, e0, e1)); v.push_back(ms * 1000.f / reps);
        }
        std::sort(v.begin(), v.end());
        printf("{\"probe\":\"exit_accounting\",\"case\":\"%s\",\"ctas\":%u,\"b2b\":%d,\"us_per_launch_p50\":%.2f,\"min\":%.2f}\n",
               names[mode], W, reps, v[v.size() / 2], v[0]);
      }
    }
  }
  return 0;
}
