// Phase-0 hardware probes. Standalone executable; not part of the
// product library. Prints one JSON object per probe on stdout.
//   1. %smid / %nsmid density and per-SM CTA counts at full occupancy
//   2. %globaltimer resolution (H3)
//   3. control-word propagation: cuStreamWriteValue32 on a high-priority stream vs a host
//      store to mapped pinned memory, observed by resident spinning CTAs (H1)
//   4. empty-kernel launch latency (host-timed) and back-to-back device gap
//   5. same-address atomicAdd throughput vs chunk size C (M2)
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <chrono>
#include <vector>
#include <algorithm>
#include <thread>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "CUDA %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); exit(1);} } while (0)

__device__ __forceinline__ uint32_t smid() { uint32_t r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }
__device__ __forceinline__ uint32_t nsmid() { uint32_t r; asm volatile("mov.u32 %0, %%nsmid;" : "=r"(r)); return r; }
__device__ __forceinline__ uint64_t gtimer() { uint64_t r; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(r)); return r; }
__device__ __forceinline__ uint32_t ld_acquire(const uint32_t* p) {
  uint32_t v; asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v; }
__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t* p) {
  uint32_t v; asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v; }

__global__ void k_smid(uint32_t* out, uint32_t* arrive, uint32_t total) {
  if (threadIdx.x == 0) {
    out[2 * blockIdx.x] = smid();
    out[2 * blockIdx.x + 1] = nsmid();
    atomicAdd(arrive, 1);
    // hold the slot until every CTA has been dispatched (proves co-residency) or timeout
    uint64_t t0 = gtimer();
    while (ld_acquire(arrive) < total && gtimer() - t0 < 200000000ull) {}
  }
  __syncthreads();
}

__global__ void k_timer(uint64_t* out, int n) {
  uint64_t last = gtimer(); int k = 0;
  uint64_t t0 = last;
  while (k < n && gtimer() - t0 < 50000000ull) {
    uint64_t t = gtimer();
    if (t != last) { out[k++] = t - last; last = t; }
  }
}

// resident spinners: every CTA's thread 0 spins on ctrl; records observe time; last one writes host flag
__global__ void k_spin(const uint32_t* ctrl, int sys, uint64_t* t_obs, uint32_t* cnt, volatile uint32_t* host_flag,
                       uint32_t total) {
  if (threadIdx.x == 0) {
    uint64_t t0 = gtimer();
    while (true) {
      uint32_t v = sys ? ld_acquire_sys(ctrl) : ld_acquire(ctrl);
      if (v) break;
      if (gtimer() - t0 > 2000000000ull) break;  // 2 s safety
    }
    t_obs[blockIdx.x] = gtimer();
    if (atomicAdd(cnt, 1) + 1 == total) {
      __threadfence_system();
      *host_flag = 1;
    }
  }
  __syncthreads();
}

__global__ void k_empty() {}
__global__ void k_stamp(uint64_t* t) { if (threadIdx.x == 0 && blockIdx.x == 0) *t = gtimer(); }

__global__ void k_atomic(uint32_t* ctr, uint32_t n_total, uint32_t C, uint32_t* sink) {
  __shared__ uint32_t s;
  uint32_t acc = 0;
  while (true) {
    if (threadIdx.x == 0) s = atomicAdd(ctr, C);
    __syncthreads();
    uint32_t v = s;
    __syncthreads();
    if (v >= n_total) break;
    acc += v;
  }
  if (acc == 0xffffffffu) *sink = acc;
}

typedef CUresult (*PFN_wv32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);

static double now_us() {
  return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

int main() {
  cudaDeviceProp prop; CK(cudaGetDeviceProperties(&prop, 0));
  printf("{\"probe\":\"device\",\"name\":\"%s\",\"sms\":%d,\"l2\":%d,\"smem_per_sm\":%zu,\"max_thr_sm\":%d,\"cc\":\"%d.%d\"}\n",
         prop.name, prop.multiProcessorCount, prop.l2CacheSize, prop.sharedMemPerMultiprocessor,
         prop.maxThreadsPerMultiProcessor, prop.major, prop.minor);
  int nsm = prop.multiProcessorCount;

  // ---- 1. smid map at full occupancy (256-thread CTAs, 8 per SM)
  {
    int per = 0; CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_smid, 256, 0));
    uint32_t total = per * nsm;
    uint32_t *d, *arr; CK(cudaMalloc(&d, 8 * total)); CK(cudaMalloc(&arr, 4)); CK(cudaMemset(arr, 0, 4));
    k_smid<<<total, 256>>>(d, arr, total); CK(cudaDeviceSynchronize());
    std::vector<uint32_t> h(2 * total); CK(cudaMemcpy(h.data(), d, 8 * total, cudaMemcpyDeviceToHost));
    uint32_t arrived; CK(cudaMemcpy(&arrived, arr, 4, cudaMemcpyDeviceToHost));
    uint32_t mx = 0, ns = 0; std::vector<int> cnt(1024, 0);
    for (uint32_t i = 0; i < total; i++) { mx = std::max(mx, h[2 * i]); ns = h[2 * i + 1]; cnt[h[2 * i]]++; }
    int distinct = 0, mn = 1 << 30, mxc = 0;
    for (uint32_t s = 0; s <= mx; s++) if (cnt[s]) { distinct++; mn = std::min(mn, cnt[s]); mxc = std::max(mxc, cnt[s]); }
    printf("{\"probe\":\"smid\",\"occ_per_sm\":%d,\"grid\":%u,\"arrived\":%u,\"max_smid\":%u,\"nsmid\":%u,\"distinct\":%d,"
           "\"min_per_sm\":%d,\"max_per_sm\":%d,\"first16\":[", per, total, arrived, mx, ns, distinct, mn, mxc);
    for (int i = 0; i < 16; i++) printf("%u%s", h[2 * i], i < 15 ? "," : "]}\n");
    CK(cudaFree(d)); CK(cudaFree(arr));
  }
  // ---- 2. globaltimer resolution
  {
    uint64_t* d; CK(cudaMalloc(&d, 8 * 4096)); CK(cudaMemset(d, 0, 8 * 4096));
    k_timer<<<1, 1>>>(d, 4096); CK(cudaDeviceSynchronize());
    std::vector<uint64_t> h(4096); CK(cudaMemcpy(h.data(), d, 8 * 4096, cudaMemcpyDeviceToHost));
    std::vector<uint64_t> v; for (auto x : h) if (x) v.push_back(x);
    std::sort(v.begin(), v.end());
    printf("{\"probe\":\"globaltimer\",\"samples\":%zu,\"min_ns\":%llu,\"p50_ns\":%llu,\"max_ns\":%llu}\n", v.size(),
           (unsigned long long)(v.empty() ? 0 : v[0]), (unsigned long long)(v.empty() ? 0 : v[v.size() / 2]),
           (unsigned long long)(v.empty() ? 0 : v.back()));
    CK(cudaFree(d));
  }
  // ---- 3. flag propagation
  {
    PFN_wv32 wv32 = nullptr; cudaDriverEntryPointQueryResult q;
    CK(cudaGetDriverEntryPoint("cuStreamWriteValue32", (void**)&wv32, cudaEnableDefault, &q));
    int lo, hi; CK(cudaDeviceGetStreamPriorityRange(&lo, &hi));
    cudaStream_t run_s, ctl_s;
    CK(cudaStreamCreateWithPriority(&run_s, cudaStreamNonBlocking, lo));
    CK(cudaStreamCreateWithPriority(&ctl_s, cudaStreamNonBlocking, hi));
    int per = 0; CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_spin, 256, 0));
    uint32_t total = per * nsm;
    uint32_t* dctrl; CK(cudaMalloc(&dctrl, 4));
    uint32_t* hctrl; CK(cudaHostAlloc(&hctrl, 4, cudaHostAllocMapped)); uint32_t* hctrl_d; CK(cudaHostGetDevicePointer(&hctrl_d, hctrl, 0));
    uint32_t* hflag; CK(cudaHostAlloc(&hflag, 4, cudaHostAllocMapped)); uint32_t* hflag_d; CK(cudaHostGetDevicePointer(&hflag_d, hflag, 0));
    uint64_t* tobs; CK(cudaMalloc(&tobs, 8 * total)); uint32_t* cnt; CK(cudaMalloc(&cnt, 4));
    uint64_t* tstamp; CK(cudaMalloc(&tstamp, 8));
    for (int mode = 0; mode < 2; mode++) {
      std::vector<double> lat_host, lat_dev_spread;
      for (int rep = 0; rep < 30; rep++) {
        CK(cudaMemset(dctrl, 0, 4)); *hctrl = 0; *(volatile uint32_t*)hflag = 0; CK(cudaMemset(cnt, 0, 4));
        CK(cudaDeviceSynchronize());
        k_spin<<<total, 256, 0, run_s>>>(mode == 0 ? dctrl : hctrl_d, mode, tobs, cnt, hflag_d, total);
        std::this_thread::sleep_for(std::chrono::milliseconds(2));
        double t0 = now_us();
        if (mode == 0) { CUresult r = wv32((CUstream)ctl_s, (CUdeviceptr)dctrl, 1, 0); if (r) { printf("wv32 err %d\n", r); return 1; } }
        else { __atomic_store_n(hctrl, 1u, __ATOMIC_RELEASE); }
        while (__atomic_load_n(hflag, __ATOMIC_ACQUIRE) == 0) {}
        double t1 = now_us();
        CK(cudaStreamSynchronize(run_s));
        std::vector<uint64_t> h(total); CK(cudaMemcpy(h.data(), tobs, 8 * total, cudaMemcpyDeviceToHost));
        auto mm = std::minmax_element(h.begin(), h.end());
        lat_host.push_back(t1 - t0); lat_dev_spread.push_back((*mm.second - *mm.first) / 1000.0);
      }
      std::sort(lat_host.begin(), lat_host.end()); std::sort(lat_dev_spread.begin(), lat_dev_spread.end());
      printf("{\"probe\":\"flag_%s\",\"workers\":%u,\"host_roundtrip_us_p50\":%.2f,\"min\":%.2f,\"max\":%.2f,"
             "\"device_observe_spread_us_p50\":%.3f}\n", mode == 0 ? "stream_memop" : "host_mapped", total,
             lat_host[15], lat_host[0], lat_host.back(), lat_dev_spread[15]);
    }
    // ---- 4. launch latency
    std::vector<double> l;
    for (int i = 0; i < 200; i++) { double t0 = now_us(); k_empty<<<1, 32, 0, run_s>>>(); CK(cudaStreamSynchronize(run_s)); l.push_back(now_us() - t0); }
    std::sort(l.begin(), l.end());
    uint64_t *ta, *tb; CK(cudaMalloc(&ta, 8)); CK(cudaMalloc(&tb, 8));
    std::vector<double> gap;
    for (int i = 0; i < 100; i++) {
      k_stamp<<<1, 32, 0, run_s>>>(ta); k_stamp<<<1, 32, 0, run_s>>>(tb); CK(cudaStreamSynchronize(run_s));
      uint64_t a, b; CK(cudaMemcpy(&a, ta, 8, cudaMemcpyDeviceToHost)); CK(cudaMemcpy(&b, tb, 8, cudaMemcpyDeviceToHost));
      gap.push_back((b - a) / 1000.0);
    }
    std::sort(gap.begin(), gap.end());
    printf("{\"probe\":\"launch\",\"empty_launch_sync_us_p50\":%.2f,\"min\":%.2f,\"b2b_device_gap_us_p50\":%.3f,\"min\":%.3f}\n",
           l[100], l[0], gap[50], gap[0]);
    // ---- 5. atomic fetch rate vs C at full occupancy
    uint32_t* ctr; CK(cudaMalloc(&ctr, 8));
    int per2 = 0; CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per2, k_atomic, 256, 0));
    for (uint32_t C : {1u, 2u, 4u, 8u, 16u, 64u}) {
      uint32_t n_total = 1u << 24;
      cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
      CK(cudaMemset(ctr, 0, 4)); k_atomic<<<per2 * nsm, 256, 0, run_s>>>(ctr, n_total, C, ctr + 1);
      CK(cudaMemsetAsync(ctr, 0, 4, run_s));
      CK(cudaEventRecord(e0, run_s)); k_atomic<<<per2 * nsm, 256, 0, run_s>>>(ctr, n_total, C, ctr + 1); CK(cudaEventRecord(e1, run_s));
      CK(cudaStreamSynchronize(run_s)); float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
      double fetches = (double)n_total / C;
      printf("{\"probe\":\"atomic_fetch\",\"C\":%u,\"workers\":%d,\"fetches_per_us\":%.1f,\"blocks_per_us\":%.1f}\n", C,
             per2 * nsm, fetches / (ms * 1000.0), n_total / (ms * 1000.0));
    }
  }
  return 0;
}
