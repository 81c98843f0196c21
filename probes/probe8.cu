// Probe 8: how fast does a host request reach a running kernel, with and without a large H2D copy
// in flight on another stream (DESIGN §8 e2e: a request memop issued during the waiting kernel's
// 67 MB input copy arrived ~20 us late)? A 1-CTA kernel spins on a flag and acknowledges each new
// value into mapped host memory; the host measures request -> acknowledgement for two transports:
//   memop  : cuStreamWriteValue32 on a separate high-priority stream to a device-memory flag
//   mapped : a plain CPU store to a pinned, mapped host word (the kernel polls it over PCIe)
#include <cuda.h>
#include <cuda_runtime.h>
#include <chrono>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#define CK(x) do { cudaError_t e = (x); if (e) { printf("CUDA %s line %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__global__ void k_spin(const volatile uint32_t* dev_flag, const volatile uint32_t* host_flag, uint32_t* ack,
                       uint32_t rounds, int use_host) {
  uint32_t seen = 0;
  for (uint32_t r = 1; r <= rounds; ++r) {
    uint32_t v;
    do {
      if (use_host) asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(host_flag));
      else asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(dev_flag));
    } while (v == seen);
    seen = v;
    asm volatile("st.relaxed.sys.global.u32 [%0], %1;" :: "l"(ack), "r"(v) : "memory");
  }
}

typedef CUresult (*PFN_wv32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);

static double now_us() {
  return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

int main() {
  PFN_wv32 wv = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuStreamWriteValue32", (void**)&wv, cudaEnableDefault, &q));
  uint32_t* dev_flag; CK(cudaMalloc(&dev_flag, 4)); CK(cudaMemset(dev_flag, 0, 4));
  uint32_t *h_flag, *h_ack, *d_hflag, *d_ack;
  CK(cudaHostAlloc(&h_flag, 64, cudaHostAllocMapped)); CK(cudaHostAlloc(&h_ack, 64, cudaHostAllocMapped));
  CK(cudaHostGetDevicePointer(&d_hflag, h_flag, 0)); CK(cudaHostGetDevicePointer(&d_ack, h_ack, 0));
  const size_t big = 64u << 20;
  void* h_big; void* d_big; CK(cudaHostAlloc(&h_big, big, 0)); CK(cudaMalloc(&d_big, big));
  int lo, hi; CK(cudaDeviceGetStreamPriorityRange(&lo, &hi));
  cudaStream_t s_k, s_ctl, s_copy;
  CK(cudaStreamCreateWithPriority(&s_k, cudaStreamNonBlocking, lo));
  CK(cudaStreamCreateWithPriority(&s_ctl, cudaStreamNonBlocking, hi));
  CK(cudaStreamCreateWithFlags(&s_copy, cudaStreamNonBlocking));
  const uint32_t rounds = 40;
  for (int use_host = 0; use_host < 2; ++use_host) {
    for (int dma = 0; dma < 2; ++dma) {
      *h_flag = 0; *h_ack = 0; CK(cudaMemset(dev_flag, 0, 4)); CK(cudaDeviceSynchronize());
      k_spin<<<1, 32, 0, s_k>>>(dev_flag, d_hflag, d_ack, rounds, use_host);
      std::vector<double> lat;
      for (uint32_t r = 1; r <= rounds; ++r) {
        if (dma) CK(cudaMemcpyAsync(d_big, h_big, big, cudaMemcpyHostToDevice, s_copy));
        const double t0 = now_us();
        if (use_host) __atomic_store_n(h_flag, r, __ATOMIC_RELEASE);
        else if (wv((CUstream)s_ctl, (CUdeviceptr)dev_flag, r, 0) != CUDA_SUCCESS) { printf("memop failed\n"); return 1; }
        while (__atomic_load_n(h_ack, __ATOMIC_ACQUIRE) != r) {}
        lat.push_back(now_us() - t0);
        CK(cudaStreamSynchronize(s_copy));
      }
      CK(cudaStreamSynchronize(s_k));
      std::sort(lat.begin(), lat.end());
      printf("{\"probe\":\"request_path\",\"transport\":\"%s\",\"h2d_copy_in_flight\":%s,\"us_p50\":%.2f,\"us_min\":%.2f,\"us_max\":%.2f}\n",
             use_host ? "mapped" : "memop", dma ? "true" : "false", lat[lat.size() / 2], lat[0], lat.back());
    }
  }
  return 0;
}
