// Probe 10: SpMV body variants on the configs[1] matrix (2^20 rows, row length uniform 0..20,
// columns uniform), unwrapped grids of 128-row blocks, L2 flushed between reps. Which body shape
// gets closest to the random-gather ceiling of probe 6 (the L1TEX->XBAR request rate)?
//   vec4      : 4 lanes per row, 8 rows per warp per pass, 2 passes per block (the VEC body)
//   vec4x2    : 4 lanes per row, both passes' rows in flight together (16 rows per warp)
//   vec2      : 2 lanes per row, 16 rows per warp, one pass
//   vec8      : 8 lanes per row, 4 rows per warp, 4 passes
//   vec4_nc   : vec4 with col/val through the non-coherent path (ld.global.nc.L1::no_allocate)
// Each variant runs with and without an L2 persisting window on x. One JSON line per case.
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <random>
#include <vector>
#define CK(x) do { cudaError_t e = (x); if (e) { printf("CUDA %s line %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

template <int LANES, int U, int PASSES_TOGETHER>
__global__ void __launch_bounds__(256, 8) spmv_vec(const int* __restrict__ rp, const int* __restrict__ col,
                                                   const float* __restrict__ val, const float* __restrict__ x,
                                                   float* __restrict__ y, int rows) {
  constexpr int RPW = 32 / LANES;                       // rows per warp per pass
  constexpr int PASSES = 128 / (8 * RPW);               // passes per 128-row block
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31, sub = lane % LANES;
#pragma unroll 1
  for (int pass0 = 0; pass0 < PASSES; pass0 += PASSES_TOGETHER) {
    int r[PASSES_TOGETHER], s[PASSES_TOGETHER], e[PASSES_TOGETHER];
    float acc[PASSES_TOGETHER];
#pragma unroll
    for (int j = 0; j < PASSES_TOGETHER; ++j) {
      r[j] = blockIdx.x * 128 + (pass0 + j) * 8 * RPW + w * RPW + lane / LANES;
      const bool v = r[j] < rows;
      s[j] = v ? __ldg(rp + r[j]) : 0;
      e[j] = v ? __ldg(rp + r[j] + 1) : 0;
      acc[j] = 0.f;
    }
    int len = 0;
#pragma unroll
    for (int j = 0; j < PASSES_TOGETHER; ++j) len = max(len, e[j] - s[j]);
    for (int o = sub; o < len; o += LANES * U) {
      int c[PASSES_TOGETHER][U];
      float vv[PASSES_TOGETHER][U];
#pragma unroll
      for (int j = 0; j < PASSES_TOGETHER; ++j)
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int q = s[j] + o + LANES * u;
          c[j][u] = q < e[j] ? __ldcs(col + q) : 0;
          vv[j][u] = q < e[j] ? __ldcs(val + q) : 0.f;
        }
#pragma unroll
      for (int j = 0; j < PASSES_TOGETHER; ++j)
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const float xv = __ldg(x + c[j][u]);
          if (s[j] + o + LANES * u < e[j]) acc[j] += vv[j][u] * xv;
        }
    }
#pragma unroll
    for (int j = 0; j < PASSES_TOGETHER; ++j) {
#pragma unroll
      for (int m = 1; m < LANES; m <<= 1) acc[j] += __shfl_xor_sync(0xffffffffu, acc[j], m);
      if (r[j] < rows && sub == 0) __stcs(y + r[j], acc[j]);
    }
  }
}

__global__ void flush_k(int4* b, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    b[i] = make_int4(1, 2, 3, (int)i);
}

int main() {
  const int rows = 1 << 20;
  std::mt19937 g(2);
  std::vector<int> rp(rows + 1, 0);
  for (int r = 0; r < rows; ++r) rp[r + 1] = rp[r] + (int)(g() % 21);
  const int nnz = rp[rows];
  std::vector<int> col(nnz);
  std::vector<float> val(nnz, 0.5f), x(rows, 1.f);
  for (int i = 0; i < nnz; ++i) col[i] = (int)(g() % rows);
  for (int r = 0; r < rows; ++r) std::sort(col.begin() + rp[r], col.begin() + rp[r + 1]);
  int *d_rp, *d_col; float *d_val, *d_x, *d_y; int4* d_fl;
  const size_t fl_n = (512u << 20) / 16;
  CK(cudaMalloc(&d_rp, (rows + 1) * 4)); CK(cudaMalloc(&d_col, nnz * 4)); CK(cudaMalloc(&d_val, nnz * 4));
  CK(cudaMalloc(&d_x, rows * 4)); CK(cudaMalloc(&d_y, rows * 4)); CK(cudaMalloc(&d_fl, fl_n * 16));
  CK(cudaMemcpy(d_rp, rp.data(), (rows + 1) * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(d_col, col.data(), nnz * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(d_val, val.data(), nnz * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(d_x, x.data(), rows * 4, cudaMemcpyHostToDevice));
  cudaStream_t s; CK(cudaStreamCreate(&s));
  cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  int maxp = 0; CK(cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, 0));
  CK(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, std::min<size_t>(maxp, 8u << 20)));
  const int nb = rows / 128;
  auto run = [&](auto kern, const char* name, bool persist) -> int {
    cudaStreamAttrValue a = {};
    if (persist) {
      a.accessPolicyWindow.base_ptr = d_x;
      a.accessPolicyWindow.num_bytes = rows * 4;
      a.accessPolicyWindow.hitRatio = 1.0f;
      a.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
      a.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    }
    CK(cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &a));
    std::vector<float> v;
    for (int r = 0; r < 40; ++r) {
      flush_k<<<148 * 8, 256, 0, s>>>(d_fl, fl_n);
      CK(cudaEventRecord(e0, s));
      kern<<<nb, 256, 0, s>>>(d_rp, d_col, d_val, d_x, d_y, rows);
      CK(cudaEventRecord(e1, s)); CK(cudaEventSynchronize(e1));
      float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
      if (r >= 5) v.push_back(ms * 1000.f);
    }
    std::sort(v.begin(), v.end());
    double mean = 0; for (size_t i = v.size() / 10; i < v.size() - v.size() / 10; ++i) mean += v[i];
    mean /= (v.size() - 2 * (v.size() / 10));
    printf("{\"probe\":\"spmv_body\",\"case\":\"%s\",\"persist_x\":%d,\"us_p50\":%.2f,\"us_mean80\":%.2f,\"us_min\":%.2f}\n",
           name, persist ? 1 : 0, v[v.size() / 2], mean, v[0]);
    if (persist) { CK(cudaCtxResetPersistingL2Cache()); }
    return 0;
  };
  for (int pers = 0; pers < 2; ++pers) {
    if (run(spmv_vec<4, 4, 1>, "vec4_U4", pers)) return 1;
    if (run(spmv_vec<4, 2, 2>, "vec4x2_U2", pers)) return 1;
    if (run(spmv_vec<4, 4, 2>, "vec4x2_U4", pers)) return 1;
    if (run(spmv_vec<2, 4, 1>, "vec2_U4", pers)) return 1;
    if (run(spmv_vec<2, 2, 1>, "vec2_U2", pers)) return 1;
    if (run(spmv_vec<8, 2, 1>, "vec8_U2", pers)) return 1;
    if (run(spmv_vec<8, 2, 2>, "vec8x2_U2", pers)) return 1;
    if (run(spmv_vec<4, 2, 1>, "vec4_U2", pers)) return 1;
  }
  return 0;
}
