// kernels.hpp — host-side dispatch table over the instantiated device kernels.
#pragma once
#include <cuda_runtime.h>
#include <cstdint>

#include "../../include/flep.h"
#include "flep_device.cuh"

namespace flep {

struct BodyOps {
  int32_t body;
  int threads;
  size_t args_size;
  // launch W worker CTAs of flep_worker<Body> on stream s
  cudaError_t (*worker)(const void* args, const WorkerParams& p, uint32_t W, cudaStream_t s, bool cov);
  // launch the original kernel: full grid (count == 0) or the 1-D slice [offset, offset+count)
  cudaError_t (*unwrapped)(const void* args, dim3 grid, uint32_t offset, uint32_t count, cudaStream_t s);
  // resident worker CTAs per SM
  cudaError_t (*occupancy)(int* ctas_per_sm, bool cov);
  // optional argument / grid validation (nullptr = none); returns a static message or nullptr
  const char* (*validate)(const void* args, dim3 grid);
  // launch the CLC variant (flep_clc_worker<Body>) over the original grid of N blocks (1-D);
  // nullptr for bodies that own their loop (GEMM)
  cudaError_t (*clc)(const void* args, const WorkerParams& p, uint32_t N, cudaStream_t s, bool cov);
  // launch W CTAs of the scheduling-warp worker (flep_worker_sw<Body>, R26) and its occupancy;
  // nullptr for bodies that own their loop or synchronise the whole CTA inside run()
  cudaError_t (*worker_sw)(const void* args, const WorkerParams& p, uint32_t W, cudaStream_t s, bool cov);
  cudaError_t (*occupancy_sw)(int* ctas_per_sm, bool cov);
  // warp-task worker (flep_warp_worker<Body>, R30): launch G CTAs (G x threads/32 warp workers)
  // and its occupancy; warp_tasks = tasks per original block (0 = the body does not decompose)
  cudaError_t (*warp_worker)(const void* args, const WorkerParams& p, uint32_t G, cudaStream_t s, bool cov);
  cudaError_t (*occupancy_warp)(int* ctas_per_sm, bool cov);
  uint32_t warp_tasks;
  // kernel slicing with the device check (flep_slice<Body>, R31): blocks [offset, offset+count)
  cudaError_t (*sliced)(const void* args, dim3 grid, uint32_t offset, uint32_t count, const SliceParams& sp,
                        cudaStream_t s);
  // the static persistent twin (flep_static<Body>, U1): `ctas` resident CTAs, chunks of C blocks
  cudaError_t (*static_launch)(const void* args, dim3 grid, uint32_t ctas, uint32_t chunk, cudaStream_t s);
  // CTA-pair bodies (R32): the worker is a cluster of 2 CTAs; max resident pairs
  cudaError_t (*max_pairs)(int* pairs, bool cov);
  // in-chunk stop worker (flep_worker_ic<Body>, R33) and its occupancy
  cudaError_t (*worker_ic)(const void* args, const WorkerParams& p, uint32_t W, cudaStream_t s, bool cov);
  cudaError_t (*occupancy_ic)(int* ctas_per_sm, bool cov);
  // in-tile accumulator spill slots of kSpillBytes per CTA (0 = 1; the wide pair tile: 2)
  uint32_t spill_per_cta;
};

const BodyOps* body_ops(int32_t body);
// user-defined bodies: the id (>= FLEP_BODY_USER_FIRST), -1 invalid table, -2 no slot left
int32_t register_user_body(const flep_body_ops* ops, const char** why);
// GEMM bodies (gemm_tcgen05.cu, gemm2_tcgen05.cu)
cudaError_t gemm_static_launch(const void* user, dim3 grid, uint32_t ctas, uint32_t chunk, cudaStream_t s);
cudaError_t gemm2_worker_launch(const void* user, const WorkerParams& p, uint32_t ctas, cudaStream_t s, bool cov);
cudaError_t gemm2_unwrapped_launch(const void* user, dim3 grid, uint32_t offset, uint32_t count, cudaStream_t s);
cudaError_t gemm2_static_launch(const void* user, dim3 grid, uint32_t ctas, uint32_t chunk, cudaStream_t s);
cudaError_t gemm2_occupancy(int* k, bool cov);
cudaError_t gemm2_slice_launch(const void* user, dim3 grid, uint32_t offset, uint32_t count, const SliceParams& sp,
                               cudaStream_t s);
cudaError_t gemm2_max_pairs(int* pairs, bool cov);
const char* gemm2_validate(const void* user, dim3 grid);
// the wide pair tile (256x512, FLEP_BODY_GEMM_BF16_2SM_W): same signatures
cudaError_t gemm2w_worker_launch(const void* user, const WorkerParams& p, uint32_t ctas, cudaStream_t s, bool cov);
cudaError_t gemm2w_unwrapped_launch(const void* user, dim3 grid, uint32_t offset, uint32_t count, cudaStream_t s);
cudaError_t gemm2w_static_launch(const void* user, dim3 grid, uint32_t ctas, uint32_t chunk, cudaStream_t s);
cudaError_t gemm2w_occupancy(int* k, bool cov);
cudaError_t gemm2w_slice_launch(const void* user, dim3 grid, uint32_t offset, uint32_t count, const SliceParams& sp,
                                cudaStream_t s);
cudaError_t gemm2w_max_pairs(int* pairs, bool cov);
const char* gemm2w_validate(const void* user, dim3 grid);
cudaError_t gemm_slice_launch(const void* user, dim3 grid, uint32_t offset, uint32_t count,
                              const SliceParams& sp, cudaStream_t s);
#ifdef FLEP_TRACE
cudaError_t set_unwrapped_trace(uint64_t* p);
#endif

template <class Body>
cudaError_t launch_worker_raw(const typename Body::Args& a, const WorkerParams& p, uint32_t W, cudaStream_t s, bool cov);
template <class Body>
cudaError_t launch_unwrapped_raw(const typename Body::Args& a, dim3 grid, uint32_t offset, uint32_t count, cudaStream_t s);
template <class Body>
cudaError_t occupancy_raw(int* k, bool cov);
template <class Body>
cudaError_t launch_static_raw(const typename Body::Args& a, dim3 grid, uint32_t ctas, uint32_t chunk, cudaStream_t s);
template <class Body>
cudaError_t launch_slice_raw(const typename Body::Args& a, dim3 grid, uint32_t offset, uint32_t count,
                             const SliceParams& sp, cudaStream_t s);
template <class Body>
cudaError_t launch_clc_raw(const typename Body::Args& a, const WorkerParams& p, uint32_t N, cudaStream_t s, bool cov);

// TMA-staged stencil body (stencil_tma.cu)
const char* stencil_tma_validate(const void* user, dim3 grid);
cudaError_t stencil_tma_worker_launch(const void* user, const WorkerParams& p, uint32_t W, cudaStream_t s, bool cov);
cudaError_t stencil_tma_unwrapped_launch(const void* user, dim3 grid, uint32_t offset, uint32_t count, cudaStream_t s);
cudaError_t stencil_tma_clc_launch(const void* user, const WorkerParams& p, uint32_t N, cudaStream_t s, bool cov);
cudaError_t stencil_tma_occupancy(int* k, bool cov);
cudaError_t stencil_tma_slice_launch(const void* user, dim3 grid, uint32_t offset, uint32_t count,
                                     const SliceParams& sp, cudaStream_t s);

}  // namespace flep
