// Probe 11: can the SpMV's random x-gather pass the L1TEX -> XBAR miss-request ceiling of probe 6
// (one request per cycle per SM) by going through the TMA unit instead of the LSU?
// Same x (f32[2^20], 4 MiB, L2-resident) and the same 10,491,315 uniform indices as probe 6.
//   lsu_U8   : probe 6's best form (each thread 8 independent __ldg gathers in flight)
//   g4_S*    : x viewed as a 2-D tensor [2^18][4] f32; every thread issues one TMA
//              cp.async.bulk.tensor.2d...tile::gather4 for 4 indices (4 rows of 16 B land in smem),
//              S stages of 1024 indices per CTA in flight, mbarrier complete_tx per stage
//   bulk_S*  : the same pipeline with one 16-B cp.async.bulk (non-tensor) per index
//   mix_S*   : half the indices by gather4, half by LSU gathers issued behind them (do the two
//              paths add?)
// Every case checks sum(x[idx]) against the host (x = i % 7, exact in double).
#include <cuda.h>
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <random>
#include <vector>
#define CK(x) do { cudaError_t e = (x); if (e) { printf("CUDA %s line %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

constexpr int kT = 256;             // threads per CTA
constexpr int kTile = kT * 4;       // indices per stage

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, int n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(n) : "memory");
}
__device__ __forceinline__ void mbar_expect_arrive(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n W%=: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W%=;\n}\n" ::"r"(smem_u32(b)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void g4(void* dst, const CUtensorMap* tm, uint64_t* bar, int r0, int r1, int r2, int r3) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4, %5, %6, %7}], [%2];" ::"r"(smem_u32(dst)),
      "l"(tm), "r"(smem_u32(bar)), "r"(0), "r"(r0), "r"(r1), "r"(r2), "r"(r3)
      : "memory");
}
__device__ __forceinline__ void bulk16(void* dst, const void* src, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 16, [%2];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(smem_u32(bar))
               : "memory");
}

__device__ __forceinline__ void block_sum(float acc, double* out) {
  __shared__ float part[kT / 32];
  for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    double s = 0;
    for (int w = 0; w < kT / 32; ++w) s += part[w];
    atomicAdd(out, s);
  }
}

template <int U>
__global__ void __launch_bounds__(kT) k_lsu(const int* __restrict__ idx, const float* __restrict__ x, double* out,
                                            int m) {
  float acc = 0.f;
  const int stride = gridDim.x * blockDim.x;
  for (int i0 = blockIdx.x * blockDim.x + threadIdx.x; i0 < m; i0 += U * stride) {
    int c[U];
#pragma unroll
    for (int u = 0; u < U; ++u) c[u] = i0 + u * stride < m ? __ldcs(idx + i0 + u * stride) : -1;
#pragma unroll
    for (int u = 0; u < U; ++u) acc += c[u] >= 0 ? __ldg(x + c[u]) : 0.f;
  }
  block_sum(acc, out);
}

// MODE 0: gather4, 1: bulk 16 B per index, 2: gather4 + as many LSU gathers behind it
template <int S, int MODE>
__global__ void __launch_bounds__(kT) k_tma(const __grid_constant__ CUtensorMap tm, const int* __restrict__ idx,
                                            const float* __restrict__ x, double* out, int m) {
  extern __shared__ __align__(128) float sbuf[];  // [S][kT][32] floats (a tensor copy's smem address is 128-B aligned)
  __shared__ __align__(8) uint64_t bar[S];
  constexpr int kPer = MODE == 2 ? 2 * kTile : kTile;  // indices consumed per stage
  const int t = threadIdx.x;
  const int ntiles = (m + kPer - 1) / kPer;
  if (t == 0)
    for (int s = 0; s < S; ++s) mbar_init(&bar[s], 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncthreads();
  float acc = 0.f;
  int c[S][4];
  auto issue = [&](int s, int tile) {
    const int base = tile * kPer + t * 4;
    int4 v = make_int4(0, 0, 0, 0);
    if (base + 3 < m) v = __ldcs(reinterpret_cast<const int4*>(idx + base));
    else {
      int* pv = &v.x;
      for (int j = 0; j < 4; ++j) pv[j] = base + j < m ? idx[base + j] : -1;
    }
    c[s][0] = v.x; c[s][1] = v.y; c[s][2] = v.z; c[s][3] = v.w;
    if (t == 0) mbar_expect_arrive(&bar[s], kT * 64);
    float* dst = sbuf + (s * kT + t) * 32;
    if (MODE == 1) {
#pragma unroll
      for (int j = 0; j < 4; ++j) bulk16(dst + 4 * j, x + (max(c[s][j], 0) & ~3), &bar[s]);
    } else {
      g4(dst, &tm, &bar[s], max(c[s][0], 0) >> 2, max(c[s][1], 0) >> 2, max(c[s][2], 0) >> 2,
         max(c[s][3], 0) >> 2);
    }
  };
  int tile = blockIdx.x, k = 0;
#pragma unroll
  for (int s = 0; s < S; ++s)
    if (tile + s * (int)gridDim.x < ntiles) issue(s, tile + s * gridDim.x);
  for (;; k ^= 1) {
    bool any = false;
#pragma unroll
    for (int s = 0; s < S; ++s) {
      if (tile >= ntiles) break;
      any = true;
      float lsu = 0.f;
      if (MODE == 2) {  // the second half of this stage's indices through the LSU while TMA is in flight
        const int base = tile * kPer + kTile + t * 4;
        int cc[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) cc[j] = base + j < m ? __ldcs(idx + base + j) : -1;
#pragma unroll
        for (int j = 0; j < 4; ++j) lsu += cc[j] >= 0 ? __ldg(x + cc[j]) : 0.f;
      }
      mbar_wait(&bar[s], k);
      const float* src = sbuf + (s * kT + t) * 32;
#pragma unroll
      for (int j = 0; j < 4; ++j) acc += c[s][j] >= 0 ? src[4 * j + (c[s][j] & 3)] : 0.f;
      acc += lsu;
      __syncthreads();
      const int nt = tile + S * gridDim.x;
      if (nt < ntiles) issue(s, nt);
      tile += gridDim.x;
    }
    if (!any || tile >= ntiles) break;
  }
  block_sum(acc, out);
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                             const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                             CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  int nsm;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  const int n = 1 << 20, m = 10491315;
  std::vector<int> h_idx(m);
  std::mt19937 g(7);
  for (int i = 0; i < m; ++i) h_idx[i] = (int)(g() % n);
  std::vector<float> h_x(n);
  for (int i = 0; i < n; ++i) h_x[i] = (float)(i % 7);
  double want = 0;
  for (int i = 0; i < m; ++i) want += h_x[h_idx[i]];
  int* idx; float* x; double* out;
  CK(cudaMalloc(&idx, m * 4)); CK(cudaMalloc(&x, n * 4)); CK(cudaMalloc(&out, 8));
  CK(cudaMemcpy(idx, h_idx.data(), m * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(x, h_x.data(), n * 4, cudaMemcpyHostToDevice));
  EncodeFn enc = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q));
  CUtensorMap tm;
  cuuint64_t dims[2] = {4, (cuuint64_t)n / 4}, strides[1] = {16};
  cuuint32_t box[2] = {4, 1}, es[2] = {1, 1};
  CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, x, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) { printf("encode failed %d\n", (int)r); return 1; }
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  auto report = [&](const char* name, int cps, std::vector<float>& v, double got) {
    std::sort(v.begin(), v.end());
    printf("{\"probe\":\"gather_paths\",\"case\":\"%s\",\"ctas_per_sm\":%d,\"us_p50\":%.2f,\"gathers_per_s\":%.4g,"
           "\"ok\":%s}\n", name, cps, v[v.size() / 2], m / (v[v.size() / 2] * 1e-6), got == want ? "true" : "false");
    fflush(stdout);
  };
  auto run_lsu = [&](auto kern, const char* name, int cps) -> int {
    std::vector<float> v; double got = 0;
    for (int rep = 0; rep < 20; ++rep) {
      CK(cudaMemset(out, 0, 8)); CK(cudaEventRecord(e0));
      kern<<<nsm * cps, kT>>>(idx, x, out, m);
      CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
      float ms; CK(cudaEventElapsedTime(&ms, e0, e1)); v.push_back(ms * 1000.f);
      CK(cudaMemcpy(&got, out, 8, cudaMemcpyDeviceToHost));
    }
    report(name, cps, v, got);
    return 0;
  };
  auto run_tma = [&](auto kern, int S, const char* name, int cps) -> int {
    const int smem = S * kT * 128;
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    std::vector<float> v; double got = 0;
    for (int rep = 0; rep < 20; ++rep) {
      CK(cudaMemset(out, 0, 8)); CK(cudaEventRecord(e0));
      kern<<<nsm * cps, kT, smem>>>(tm, idx, x, out, m);
      CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
      float ms; CK(cudaEventElapsedTime(&ms, e0, e1)); v.push_back(ms * 1000.f);
      CK(cudaMemcpy(&got, out, 8, cudaMemcpyDeviceToHost));
    }
    report(name, cps, v, got);
    return 0;
  };
  for (int cps : {4, 8}) run_lsu(k_lsu<8>, "lsu_U8", cps);
  for (int cps : {1, 2, 3}) {
    if (run_tma(k_tma<2, 0>, 2, "g4_S2", cps)) return 1;
    if (run_tma(k_tma<4, 0>, 4, "g4_S4", cps)) return 1;
    if (cps <= 2 && run_tma(k_tma<6, 0>, 6, "g4_S6", cps)) return 1;
    if (run_tma(k_tma<2, 1>, 2, "bulk_S2", cps)) return 1;
    if (run_tma(k_tma<4, 1>, 4, "bulk_S4", cps)) return 1;
    if (run_tma(k_tma<2, 2>, 2, "mix_S2", cps)) return 1;
    if (run_tma(k_tma<4, 2>, 4, "mix_S4", cps)) return 1;
  }
  return 0;
}
