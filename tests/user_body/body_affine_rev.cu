// A user-defined body for tests/test_gpu_user_body.py (the flep_register_body extension,
// include/flep_body.cuh): block b of n int32 elements (512 per block, 128 threads x 4) stages its
// x window in shared memory and writes y[i] = a * x[mirror(i)] + c * b (mod 2^32), mirror(i) =
// b*512 + 511 - (i - b*512), x beyond n read as 0. A barrier inside the body and a result that
// depends on the block index make a lost or doubled block visible in y.
#include <cstdint>

#include "flep_body.cuh"

struct AffineRevArgs {
  int32_t* y;
  const int32_t* x;
  int32_t a, c;
  uint32_t n;
};

struct AffineRevBody : flep::UserBody {
  using Args = AffineRevArgs;
  static constexpr int kThreads = 128;
  static constexpr int kMinBlocks = 16;    // the original grid's 2048 threads per SM: the worker keeps them
  static constexpr uint32_t kPer = 512;
  __device__ static void run(const Args& g, uint32_t b0, uint32_t b1, uint32_t, uint32_t) {
    __shared__ int32_t s[kPer];
    for (uint32_t b = b0; b < b1; ++b) {
      const uint32_t base = b * kPer;
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k) {
        const uint32_t j = threadIdx.x + k * kThreads;
        s[j] = base + j < g.n ? g.x[base + j] : 0;
      }
      __syncthreads();
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k) {
        const uint32_t j = threadIdx.x + k * kThreads;
        if (base + j < g.n)
          g.y[base + j] = (int32_t)((uint32_t)g.a * (uint32_t)s[kPer - 1 - j] + (uint32_t)g.c * b);
      }
      __syncthreads();                 // s is rewritten by the next block of this CTA
    }
  }
};

FLEP_DEFINE_BODY(affine_rev, AffineRevBody)
