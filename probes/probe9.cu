// Probe 9: does an L2 persisting access-policy window on x help the SpMV gathers?
// Same matrix shape as configs[1] (2^20 rows, row length uniform 0..20, columns uniform), a
// CSR-vector SpMV (4 lanes per row) and the random-gather kernel of probe 6, each timed with L2
// flushed between reps (512 MB write), without and with a persisting window over x (4 MiB,
// hitRatio 1) on the launching stream. Prints one JSON line per case.
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <random>
#include <vector>
#define CK(x) do { cudaError_t e = (x); if (e) { printf("CUDA %s line %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__global__ void __launch_bounds__(256) spmv_vec(const int* __restrict__ rp, const int* __restrict__ col,
                                                const float* __restrict__ val, const float* __restrict__ x,
                                                float* __restrict__ y, int rows) {
  const int r = blockIdx.x * 64 + (threadIdx.x >> 2), sub = threadIdx.x & 3;
  if (r >= rows) return;
  const int s = rp[r], e = rp[r + 1];
  float acc = 0.f;
  for (int p = s + sub; p < e; p += 16) {
    int c[4]; float v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) { const int q = p + 4 * u; c[u] = q < e ? __ldcs(col + q) : 0; v[u] = q < e ? __ldcs(val + q) : 0.f; }
#pragma unroll
    for (int u = 0; u < 4; ++u) acc += v[u] * __ldg(x + c[u]);
  }
  acc += __shfl_xor_sync(0xffffffffu, acc, 1);
  acc += __shfl_xor_sync(0xffffffffu, acc, 2);
  if (sub == 0) y[r] = acc;
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
  std::vector<int> col(nnz); std::vector<float> val(nnz, 0.5f), x(rows, 1.f);
  for (int i = 0; i < nnz; ++i) col[i] = (int)(g() % rows);
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
  auto run = [&](const char* name, bool persist) -> int {
    cudaStreamAttrValue a = {};
    if (persist) {
      CK(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, std::min<size_t>(maxp, 8u << 20)));
      a.accessPolicyWindow.base_ptr = d_x;
      a.accessPolicyWindow.num_bytes = rows * 4;
      a.accessPolicyWindow.hitRatio = 1.0f;
      a.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
      a.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    } else {
      a.accessPolicyWindow.num_bytes = 0;
    }
    CK(cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &a));
    std::vector<float> v;
    for (int r = 0; r < 30; ++r) {
      flush_k<<<148 * 8, 256, 0, s>>>(d_fl, fl_n);
      CK(cudaEventRecord(e0, s));
      spmv_vec<<<(rows + 63) / 64, 256, 0, s>>>(d_rp, d_col, d_val, d_x, d_y, rows);
      CK(cudaEventRecord(e1, s)); CK(cudaEventSynchronize(e1));
      float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
      if (r >= 5) v.push_back(ms * 1000.f);
    }
    std::sort(v.begin(), v.end());
    printf("{\"probe\":\"l2_persist_x\",\"case\":\"%s\",\"nnz\":%d,\"us_p50\":%.2f,\"us_min\":%.2f,\"max_persist_bytes\":%d}\n",
           name, nnz, v[v.size() / 2], v[0], maxp);
    if (persist) { CK(cudaCtxResetPersistingL2Cache()); }
    return 0;
  };
  if (run("csr_vector_no_window", false)) return 1;
  if (run("csr_vector_x_persisting", true)) return 1;
  if (run("csr_vector_no_window_again", false)) return 1;
  return 0;
}
