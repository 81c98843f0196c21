// stencil_tma.cu — host side of the TMA-staged stencil body: tensor maps (cuTensorMapEncodeTiled
// through the runtime's driver entry point), validation, launch wrappers.
#include <cuda.h>
#include <cuda_runtime.h>

#include "stencil_tma.cuh"
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

// fp32 row-major [n][n]; box {bw cols, bh rows}; out-of-range cells read as zero, clipped on store
bool make_map(CUtensorMap* m, const void* ptr, uint64_t n, uint32_t bw, uint32_t bh) {
  PFN_encode enc = encoder();
  if (!enc) return false;
  const cuuint64_t dims[2] = {n, n};
  const cuuint64_t strides[1] = {n * 4};
  const cuuint32_t box[2] = {bw, bh};
  const cuuint32_t estr[2] = {1, 1};
  return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<void*>(ptr), dims, strides, box, estr,
             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

bool to_dev(const void* user, StencilTmaArgsDev* d) {
  const flep_stencil_args& u = *reinterpret_cast<const flep_stencil_args*>(user);
  d->n = u.n;
  return make_map(&d->tma_in, u.in, u.n, Stencil5TmaBody::kInW, Stencil5TmaBody::kInH) &&
         make_map(&d->tma_out, u.out, u.n, Stencil5TmaBody::kTile, Stencil5TmaBody::kTile);
}

}  // namespace

const char* stencil_tma_validate(const void* user, dim3 grid) {
  const flep_stencil_args& u = *reinterpret_cast<const flep_stencil_args*>(user);
  if (!u.in || !u.out) return "stencil (TMA): NULL pointer";
  if (u.n < 4 || u.n % 4) return "stencil (TMA): needs n % 4 == 0 (16-byte row stride)";
  const uint32_t t = (u.n + 63) / 64;
  if (grid.x != t || grid.y != t || grid.z != 1) return "stencil (TMA): grid must be (ceil(n/64), ceil(n/64), 1)";
  if (((uintptr_t)u.in | (uintptr_t)u.out) & 15u) return "stencil (TMA): in/out must be 16-byte aligned";
  if (!encoder()) return "stencil (TMA): cuTensorMapEncodeTiled unavailable";
  return nullptr;
}

cudaError_t stencil_tma_worker_launch(const void* user, const WorkerParams& p, uint32_t W, cudaStream_t s, bool cov) {
  StencilTmaArgsDev d;
  if (!to_dev(user, &d)) return cudaErrorInvalidValue;
  return launch_worker_raw<Stencil5TmaBody>(d, p, W, s, cov);
}

cudaError_t stencil_tma_unwrapped_launch(const void* user, dim3 grid, uint32_t offset, uint32_t count, cudaStream_t s) {
  StencilTmaArgsDev d;
  if (!to_dev(user, &d)) return cudaErrorInvalidValue;
  return launch_unwrapped_raw<Stencil5TmaBody>(d, grid, offset, count, s);
}

cudaError_t stencil_tma_clc_launch(const void* user, const WorkerParams& p, uint32_t N, cudaStream_t s, bool cov) {
  StencilTmaArgsDev d;
  if (!to_dev(user, &d)) return cudaErrorInvalidValue;
  return launch_clc_raw<Stencil5TmaBody>(d, p, N, s, cov);
}

cudaError_t stencil_tma_occupancy(int* k, bool cov) { return occupancy_raw<Stencil5TmaBody>(k, cov); }

cudaError_t stencil_tma_slice_launch(const void* user, dim3 grid, uint32_t offset, uint32_t count,
                               const SliceParams& sp, cudaStream_t s) {
  StencilTmaArgsDev d;
  if (!to_dev(user, &d)) return cudaErrorInvalidValue;
  return launch_slice_raw<Stencil5TmaBody>(d, grid, offset, count, sp, s);
}

}  // namespace flep
