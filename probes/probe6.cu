// Probe 6: the random-gather ceiling that bounds the SpMV body. x is f32[2^20]
// (4 MiB, L2-resident after the first touch); idx is i32[M] uniform over [0, 2^20) read coalesced
// (like CSR col[]); each thread gathers x[idx[i]] for U independent i in flight and accumulates.
// Reports gathers/s for several occupancies / unroll depths (best = the measured gather peak),
// plus the same with 8 B of coalesced streaming per gather (col + val, the SpMV's other reads).
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <random>
#define CK(x) do { cudaError_t e = (x); if (e) { printf("CUDA %s line %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

template <int U, bool kVal>
__global__ void __launch_bounds__(256) k_gather(const int* __restrict__ idx, const float* __restrict__ val,
                                                const float* __restrict__ x, float* out, int m) {
  float acc = 0.f;
  const int stride = gridDim.x * blockDim.x;
  for (int i0 = blockIdx.x * blockDim.x + threadIdx.x; i0 < m; i0 += U * stride) {
    int c[U]; float v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int i = i0 + u * stride;
      c[u] = i < m ? __ldcs(idx + i) : 0;
      v[u] = (kVal && i < m) ? __ldcs(val + i) : 1.f;
    }
#pragma unroll
    for (int u = 0; u < U; ++u) acc += v[u] * __ldg(x + c[u]);
  }
  if (acc == 12345.f) out[0] = acc;
}

int main() {
  int nsm; CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  const int n = 1 << 20, m = 10491315;           // the SpMV's x size and nnz (configs[1])
  std::vector<int> h_idx(m); std::mt19937 g(7);
  for (int i = 0; i < m; ++i) h_idx[i] = (int)(g() % n);
  int* idx; float *x, *val, *out;
  CK(cudaMalloc(&idx, m * 4)); CK(cudaMalloc(&val, m * 4)); CK(cudaMalloc(&x, n * 4)); CK(cudaMalloc(&out, 4));
  CK(cudaMemcpy(idx, h_idx.data(), m * 4, cudaMemcpyHostToDevice));
  CK(cudaMemset(x, 0, n * 4)); CK(cudaMemset(val, 0, m * 4));
  cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  auto run = [&](auto kern, const char* name, int ctas_per_sm) -> int {
    std::vector<float> v;
    for (int r = 0; r < 20; ++r) {
      CK(cudaEventRecord(e0));
      kern<<<nsm * ctas_per_sm, 256>>>(idx, val, x, out, m);
      CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
      float ms; CK(cudaEventElapsedTime(&ms, e0, e1)); v.push_back(ms * 1000.f);
    }
    std::sort(v.begin(), v.end());
    printf("{\"probe\":\"gather_ceiling\",\"case\":\"%s\",\"ctas_per_sm\":%d,\"us_p50\":%.2f,\"gathers_per_s\":%.4g}\n",
           name, ctas_per_sm, v[v.size() / 2], m / (v[v.size() / 2] * 1e-6));
    return 0;
  };
  for (int c : {4, 8}) {
    run(k_gather<4, false>, "idx_only_U4", c);
    run(k_gather<8, false>, "idx_only_U8", c);
    run(k_gather<4, true>, "idx_val_U4", c);
    run(k_gather<8, true>, "idx_val_U8", c);
  }
  return 0;
}
