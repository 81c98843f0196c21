// gemm_tcgen05.cu — host side of the GEMM body: TMA tensor maps (cuTensorMapEncodeTiled through
// the runtime's driver entry point), argument validation, launch wrappers.
#include <cuda.h>
#include <cuda_runtime.h>

#include "gemm_tcgen05.cuh"
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

// 2-D bf16 row-major matrix [rows, cols] → box {64 cols, box_rows rows}, 128-B swizzle.
bool make_map(CUtensorMap* m, const void* ptr, uint64_t rows, uint64_t cols, uint32_t box_rows) {
  PFN_encode enc = encoder();
  if (!enc) return false;
  const cuuint64_t dims[2] = {cols, rows};
  const cuuint64_t strides[1] = {cols * 2};
  const cuuint32_t box[2] = {64, box_rows};
  const cuuint32_t estr[2] = {1, 1};
  return enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(ptr), dims, strides, box, estr,
             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

bool to_dev(const void* user, GemmArgsDev* d) {
  const flep_gemm_args& u = *reinterpret_cast<const flep_gemm_args*>(user);
  d->c = reinterpret_cast<__nv_bfloat16*>(u.c);
  d->m = u.m; d->n = u.n; d->k = u.k;
  return make_map(&d->tma_a, u.a, u.m, u.k, GemmBody::BM) && make_map(&d->tma_b, u.b, u.n, u.k, GemmBody::BN) &&
         make_map(&d->tma_c, u.c, u.m, u.n, 32);     // epilogue: 32 rows x 64 columns per bulk store
}

}  // namespace

const char* gemm_validate(const void* user, dim3 grid) {
  const flep_gemm_args& u = *reinterpret_cast<const flep_gemm_args*>(user);
  if (!u.a || !u.b || !u.c) return "GEMM: NULL matrix pointer";
  if (u.m == 0 || u.n == 0 || u.k == 0) return "GEMM: empty problem";
  if (u.m % GemmBody::BM || u.n % GemmBody::BN || u.k % GemmBody::BK) return "GEMM: needs M%128 == N%256 == K%64 == 0";
  if (grid.x != u.n / GemmBody::BN || grid.y != u.m / GemmBody::BM || grid.z != 1)
    return "GEMM: grid must be (N/256, M/128, 1)";
  if (((uintptr_t)u.a | (uintptr_t)u.b) & 15u) return "GEMM: A and B must be 16-byte aligned";
  if ((uintptr_t)u.c & 15u) return "GEMM: C must be 16-byte aligned";
  if (!encoder()) return "GEMM: cuTensorMapEncodeTiled unavailable";
  return nullptr;
}

cudaError_t gemm_worker_launch(const void* user, const WorkerParams& p, uint32_t W, cudaStream_t s, bool cov) {
  GemmArgsDev d;
  if (!to_dev(user, &d)) return cudaErrorInvalidValue;
  return launch_worker_raw<GemmBody>(d, p, W, s, cov);
}

cudaError_t gemm_unwrapped_launch(const void* user, dim3 grid, uint32_t offset, uint32_t count, cudaStream_t s) {
  GemmArgsDev d;
  if (!to_dev(user, &d)) return cudaErrorInvalidValue;
  return launch_unwrapped_raw<GemmBody>(d, grid, offset, count, s);
}

cudaError_t gemm_occupancy(int* k, bool cov) { return occupancy_raw<GemmBody>(k, cov); }

cudaError_t gemm_static_launch(const void* user, dim3 grid, uint32_t ctas, uint32_t chunk, cudaStream_t s) {
  GemmArgsDev d;
  if (!to_dev(user, &d)) return cudaErrorInvalidValue;
  return launch_static_raw<GemmBody>(d, grid, ctas, chunk, s);
}

cudaError_t gemm_slice_launch(const void* user, dim3 grid, uint32_t offset, uint32_t count,
                               const SliceParams& sp, cudaStream_t s) {
  GemmArgsDev d;
  if (!to_dev(user, &d)) return cudaErrorInvalidValue;
  return launch_slice_raw<GemmBody>(d, grid, offset, count, sp, s);
}

}  // namespace flep
