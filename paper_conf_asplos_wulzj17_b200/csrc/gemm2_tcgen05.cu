// gemm2_tcgen05.cu — host side of the CTA-pair GEMM body (gemm2_tcgen05.cuh): tensor maps
// (128-row boxes for both operands: each CTA of a pair loads its half of A and its B boxes), argument
// validation, launch wrappers (the kernels carry __cluster_dims__(2, 1, 1)).
#include <cuda.h>
#include <cuda_runtime.h>

#include "gemm2_tcgen05.cuh"
#include "kernels.hpp"

namespace flep {

namespace {

typedef CUresult (*PFN_encode)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                               const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                               CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

PFN_encode encoder() {
  static PFN_encode fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&fn, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      fn = nullptr;
  }
  return fn;
}

bool make_map(CUtensorMap* m, const void* ptr, uint64_t rows, uint64_t cols, uint32_t box_rows) {
  PFN_encode enc = encoder();
  if (!enc) return false;
  const cuuint64_t dims[2] = {cols, rows};
  const cuuint64_t strides[1] = {cols * 2};
  const cuuint32_t box[2] = {64, box_rows};     // 64 bf16 = one 128-B swizzle row
  const cuuint32_t estr[2] = {1, 1};
  return enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(ptr), dims, strides, box, estr,
             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

template <class G>
bool to_dev(const void* user, Gemm2Args* d) {
  const flep_gemm_args& u = *reinterpret_cast<const flep_gemm_args*>(user);
  d->c = reinterpret_cast<__nv_bfloat16*>(u.c);
  d->m = u.m; d->n = u.n; d->k = u.k;
  return make_map(&d->tma_a, u.a, u.m, u.k, G::BM) && make_map(&d->tma_b, u.b, u.n, u.k, 128) &&
         make_map(&d->tma_c, u.c, u.m, u.n, 32);     // epilogue: 32 rows x 64 columns per store
}

template <class G, class K>
cudaError_t smem_attr(K kern) {
  return cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)G::kDynSmem);
}

template <class G>
const char* validate(const void* user, dim3 grid) {
  const flep_gemm_args& u = *reinterpret_cast<const flep_gemm_args*>(user);
  if (!u.a || !u.b || !u.c) return "GEMM: NULL matrix pointer";
  if (u.m == 0 || u.n == 0 || u.k == 0) return "GEMM: empty problem";
  if (G::BN == 256) {
    if (u.m % G::TM || u.n % G::BN || u.k % G::BK) return "GEMM (2SM): needs M%256 == N%256 == K%64 == 0";
    if (grid.x != u.n / G::BN || grid.y != u.m / G::TM || grid.z != 1)
      return "GEMM (2SM): grid must be (N/256, M/256, 1)";
  } else {
    if (u.m % G::TM || u.n % G::BN || u.k % G::BK) return "GEMM (2SM wide): needs M%256 == N%512 == K%64 == 0";
    if (grid.x != u.n / G::BN || grid.y != u.m / G::TM || grid.z != 1)
      return "GEMM (2SM wide): grid must be (N/512, M/256, 1)";
  }
  if (((uintptr_t)u.a | (uintptr_t)u.b | (uintptr_t)u.c) & 15u) return "GEMM: A, B and C must be 16-byte aligned";
  if (!encoder()) return "GEMM: cuTensorMapEncodeTiled unavailable";
  return nullptr;
}

template <class G>
cudaError_t worker_launch(const void* user, const WorkerParams& p, uint32_t ctas, cudaStream_t s, bool cov) {
  Gemm2Args d;
  if (!to_dev<G>(user, &d)) return cudaErrorInvalidValue;
  cudaError_t e;
  if (cov) {
    if ((e = smem_attr<G>(flep_gemm2_worker<G, true>))) return e;
    flep_gemm2_worker<G, true><<<ctas, G::kThreads, G::kDynSmem, s>>>(d, p);
  } else {
    if ((e = smem_attr<G>(flep_gemm2_worker<G, false>))) return e;
    flep_gemm2_worker<G, false><<<ctas, G::kThreads, G::kDynSmem, s>>>(d, p);
  }
  return cudaGetLastError();
}

template <class G>
cudaError_t unwrapped_launch(const void* user, dim3 grid, uint32_t offset, uint32_t count, cudaStream_t s) {
  Gemm2Args d;
  if (!to_dev<G>(user, &d)) return cudaErrorInvalidValue;
  cudaError_t e = smem_attr<G>(flep_gemm2_unwrapped<G>);
  if (e) return e;
  if (count == 0) flep_gemm2_unwrapped<G><<<dim3(2 * grid.x, grid.y), G::kThreads, G::kDynSmem, s>>>(d, grid.x, grid.y, 0);
  else flep_gemm2_unwrapped<G><<<2 * count, G::kThreads, G::kDynSmem, s>>>(d, grid.x, grid.y, offset);
  return cudaGetLastError();
}

template <class G>
cudaError_t static_launch(const void* user, dim3 grid, uint32_t ctas, uint32_t /*chunk: one tile*/, cudaStream_t s) {
  Gemm2Args d;
  if (!to_dev<G>(user, &d)) return cudaErrorInvalidValue;
  cudaError_t e = smem_attr<G>(flep_gemm2_static<G>);
  if (e) return e;
  flep_gemm2_static<G><<<ctas & ~1u, G::kThreads, G::kDynSmem, s>>>(d, grid.x, grid.y, grid.x * grid.y);
  return cudaGetLastError();
}

template <class G>
cudaError_t slice_launch(const void* user, dim3 grid, uint32_t offset, uint32_t count, const SliceParams& sp,
                         cudaStream_t s) {
  Gemm2Args d;
  if (!to_dev<G>(user, &d)) return cudaErrorInvalidValue;
  cudaError_t e = smem_attr<G>(flep_gemm2_slice<G>);
  if (e) return e;
  flep_gemm2_slice<G><<<2 * count, G::kThreads, G::kDynSmem, s>>>(d, grid.x, grid.y, offset, sp);
  return cudaGetLastError();
}

template <class G>
cudaError_t occupancy(int* k, bool cov) {
  // one CTA per SM; the runtime sizes the grid in pairs (max_pairs)
  cudaError_t e = cov ? smem_attr<G>(flep_gemm2_worker<G, true>) : smem_attr<G>(flep_gemm2_worker<G, false>);
  if (e) return e;
  *k = 1;
  return cudaSuccess;
}

template <class G>
cudaError_t max_pairs(int* pairs, bool cov) {
  cudaError_t e = cov ? smem_attr<G>(flep_gemm2_worker<G, true>) : smem_attr<G>(flep_gemm2_worker<G, false>);
  if (e) return e;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(2, 1, 1);
  cfg.blockDim = dim3(G::kThreads, 1, 1);
  cfg.dynamicSmemBytes = G::kDynSmem;
  cudaLaunchAttribute attr;
  attr.id = cudaLaunchAttributeClusterDimension;
  attr.val.clusterDim.x = 2; attr.val.clusterDim.y = 1; attr.val.clusterDim.z = 1;
  cfg.attrs = &attr;
  cfg.numAttrs = 1;
  return cov ? cudaOccupancyMaxActiveClusters(pairs, flep_gemm2_worker<G, true>, &cfg)
             : cudaOccupancyMaxActiveClusters(pairs, flep_gemm2_worker<G, false>, &cfg);
}

}  // namespace

// FLEP_BODY_GEMM_BF16_2SM (256x256 pair tiles)
const char* gemm2_validate(const void* u, dim3 g) { return validate<Gemm2>(u, g); }
cudaError_t gemm2_worker_launch(const void* u, const WorkerParams& p, uint32_t c, cudaStream_t s, bool cov) {
  return worker_launch<Gemm2>(u, p, c, s, cov);
}
cudaError_t gemm2_unwrapped_launch(const void* u, dim3 g, uint32_t o, uint32_t c, cudaStream_t s) {
  return unwrapped_launch<Gemm2>(u, g, o, c, s);
}
cudaError_t gemm2_static_launch(const void* u, dim3 g, uint32_t c, uint32_t ch, cudaStream_t s) {
  return static_launch<Gemm2>(u, g, c, ch, s);
}
cudaError_t gemm2_slice_launch(const void* u, dim3 g, uint32_t o, uint32_t c, const SliceParams& sp, cudaStream_t s) {
  return slice_launch<Gemm2>(u, g, o, c, sp, s);
}
cudaError_t gemm2_occupancy(int* k, bool cov) { return occupancy<Gemm2>(k, cov); }
cudaError_t gemm2_max_pairs(int* p, bool cov) { return max_pairs<Gemm2>(p, cov); }

// FLEP_BODY_GEMM_BF16_2SM_W (256x512 pair tiles)
const char* gemm2w_validate(const void* u, dim3 g) { return validate<Gemm2W>(u, g); }
cudaError_t gemm2w_worker_launch(const void* u, const WorkerParams& p, uint32_t c, cudaStream_t s, bool cov) {
  return worker_launch<Gemm2W>(u, p, c, s, cov);
}
cudaError_t gemm2w_unwrapped_launch(const void* u, dim3 g, uint32_t o, uint32_t c, cudaStream_t s) {
  return unwrapped_launch<Gemm2W>(u, g, o, c, s);
}
cudaError_t gemm2w_static_launch(const void* u, dim3 g, uint32_t c, uint32_t ch, cudaStream_t s) {
  return static_launch<Gemm2W>(u, g, c, ch, s);
}
cudaError_t gemm2w_slice_launch(const void* u, dim3 g, uint32_t o, uint32_t c, const SliceParams& sp, cudaStream_t s) {
  return slice_launch<Gemm2W>(u, g, o, c, sp, s);
}
cudaError_t gemm2w_occupancy(int* k, bool cov) { return occupancy<Gemm2W>(k, cov); }
cudaError_t gemm2w_max_pairs(int* p, bool cov) { return max_pairs<Gemm2W>(p, cov); }

}  // namespace flep
