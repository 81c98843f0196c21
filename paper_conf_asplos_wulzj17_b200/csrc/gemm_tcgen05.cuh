// gemm_tcgen05.cuh — placeholder until the tcgen05 GEMM body lands.
#pragma once
#include <cuda_runtime.h>
#include "flep_device.cuh"

namespace flep {

struct GemmBody {
  static constexpr int kThreads = 256;
  static constexpr int kMinBlocks = 1;
};

inline cudaError_t gemm_worker_launch(const void*, const WorkerParams&, uint32_t, cudaStream_t, bool) {
  return cudaErrorNotSupported;
}
inline cudaError_t gemm_unwrapped_launch(const void*, dim3, uint32_t, uint32_t, cudaStream_t) {
  return cudaErrorNotSupported;
}
inline cudaError_t gemm_occupancy(int* k, bool) { *k = 1; return cudaSuccess; }
inline const char* gemm_validate(const void*, dim3) { return "GEMM body not built yet"; }

}  // namespace flep
