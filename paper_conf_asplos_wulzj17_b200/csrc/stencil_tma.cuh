// stencil_tma.cuh — TMA-staged 5-point stencil body (FLEP_BODY_STENCIL5_F32_TMA; same operation
// as Stencil5Body<false>). Per original block (64x64 output tile):
//   one elected thread loads the tile and its halo (rows r0-1..r0+64, columns c0-4..c0+67: a
//   72x66 fp32 box, out-of-range cells zero-filled by the TMA unit) into shared memory with
//   cp.async.bulk.tensor (mbarrier completion), the next tile of a chunk into a second buffer
//   while the current one is computed; every thread computes a 4x4 patch from shared
//   memory into an output tile in shared memory; the elected thread writes the tile back with a
//   bulk tensor store (out-of-range cells clipped by the TMA unit).
// No thread keeps a register bound to a pending global store (the stores are the TMA unit's),
// and global traffic is one bulk request per tile each way. Boundary rows/columns copy through.
#pragma once
#include <cuda.h>
#include <cstdint>
#include "flep_device.cuh"

namespace flep {

struct StencilTmaArgsDev {
  CUtensorMap tma_in;    // fp32 [n][n], box {72 cols, 66 rows}
  CUtensorMap tma_out;   // fp32 [n][n], box {64 cols, 64 rows}
  uint32_t n;
};

struct Stencil5TmaBody {
  static constexpr bool kPersistent = false;
  static constexpr int kThreads = 256;
  static constexpr int kMinBlocks = 4;
  static constexpr uint32_t kTile = 64, kInW = 72, kInH = 66;
  static constexpr uint32_t kInBytes = kInW * kInH * 4;              // 19008
  static constexpr uint32_t kInAlloc = (kInBytes + 127u) & ~127u;    // 19072
  static constexpr uint32_t kOutBytes = kTile * kTile * 4;           // 16384
  // layout (128-B aligned): [barriers, phase: 128 B][input 0][output tile][input 1]; a launch whose
  // chunks hold one block (the unwrapped grid, C = 1 workers) allocates no second input buffer,
  // which keeps more CTAs (and L1) per SM
  static constexpr size_t kDynSmem = 128 + 128 + 2 * kInAlloc + kOutBytes;
  __host__ __device__ static constexpr size_t dyn_smem(uint32_t chunk) {
    return chunk > 1 ? kDynSmem : kDynSmem - kInAlloc;
  }
  using Args = StencilTmaArgsDev;

  __device__ static uint8_t* base() {
    extern __shared__ uint8_t dsmem[];
    const uint32_t a = static_cast<uint32_t>(__cvta_generic_to_shared(dsmem));
    return dsmem + (((a + 127u) & ~127u) - a);
  }
  // two input buffers (the next tile of a chunk loads while this one is computed), one output tile
  __device__ static uint64_t* mbar(uint32_t i) { return reinterpret_cast<uint64_t*>(base()) + i; }
  __device__ static uint32_t* phase() { return reinterpret_cast<uint32_t*>(base() + 16); }
  __device__ static float* in_s(uint32_t i) {
    return reinterpret_cast<float*>(base() + 128 + (i ? kInAlloc + kOutBytes : 0u));
  }
  __device__ static float* out_s() { return reinterpret_cast<float*>(base() + 128 + kInAlloc); }
  __device__ static uint32_t u32(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }

  template <class A> __device__ static void setup(const A&) {
    if (threadIdx.x == 0) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(u32(mbar(0))) : "memory");
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(u32(mbar(1))) : "memory");
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
      *phase() = 0;                  // bit i: parity of buffer i's next completion
    }
    __syncthreads();
  }
  template <class A> __device__ static void teardown(const A&) {
    // the last tile's bulk store must have finished reading shared memory before the CTA leaves
    if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
  template <class A> __device__ static void persistent(const A&, const WorkerParams&, WorkerShared&) {}

  __device__ __forceinline__ static float cell(float c, float n, float s, float w, float e) {
    return 0.5f * c + 0.125f * (((n + s) + w) + e);
  }

  __device__ static void load(const Args& g, uint32_t b, uint32_t gx, uint32_t i) {
    const int32_t r0 = (int32_t)((b / gx) * kTile), c0 = (int32_t)((b % gx) * kTile);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(u32(mbar(i))), "r"(kInBytes) : "memory");
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
        :: "r"(u32(in_s(i))), "l"(reinterpret_cast<uint64_t>(&g.tma_in)), "r"(u32(mbar(i))), "r"(c0 - 4), "r"(r0 - 1)
        : "memory");
  }

  __device__ static void run(const Args& g, uint32_t b0, uint32_t b1, uint32_t gx, uint32_t) {
    const uint32_t tid = threadIdx.x;
    const uint32_t n = g.n;
    float* out = out_s();
    uint32_t ph = *phase();
    const uint32_t q = tid & 15u, rg = tid >> 4;                        // 16 strips x 16 row groups
    if (tid == 0) load(g, b0, gx, 0);                                  // buffer 0 is free here
    for (uint32_t b = b0; b < b1; ++b) {
      const uint32_t i = (b - b0) & 1u;
      const uint32_t tx = b % gx, ty = b / gx;
      const int32_t r0 = (int32_t)(ty * kTile), c0 = (int32_t)(tx * kTile);
      if (tid == 0) {
        // the next tile of the chunk loads into the other buffer while this one is computed (its
        // previous contents were last read before the previous tile's second barrier)
        if (b + 1 < b1) load(g, b + 1, gx, i ^ 1u);
        // the previous tile's bulk store must be done reading the output tile
        asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
      }
      __syncthreads();
      asm volatile(
          "{\n .reg .pred p;\n W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W;\n}\n"
          :: "r"(u32(mbar(i))), "r"((ph >> i) & 1u) : "memory");
      ph ^= 1u << i;
      const float* in = in_s(i);
      // thread (q, rg): columns c0+4q..+3 (smem column 4+4q), rows r0+4rg..+3 (smem row 1+4rg)
      const uint32_t jc = 4u + 4u * q;
      const uint32_t c = (uint32_t)c0 + 4u * q;
      float4 R[6];
#pragma unroll
      for (int k = 0; k < 6; ++k) R[k] = *reinterpret_cast<const float4*>(in + (4u * rg + k) * kInW + jc);
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const uint32_t r = (uint32_t)r0 + 4u * rg + k;
        const float wv = in[(4u * rg + 1 + k) * kInW + jc - 1], ev = in[(4u * rg + 1 + k) * kInW + jc + 4];
        const float4 C = R[k + 1], N = R[k], S = R[k + 2];
        float4 O;
        if (r == 0 || r + 1 == n) {
          O = C;
        } else {
          O.x = (c == 0) ? C.x : cell(C.x, N.x, S.x, wv, C.y);
          O.y = cell(C.y, N.y, S.y, C.x, C.z);
          O.z = cell(C.z, N.z, S.z, C.y, C.w);
          O.w = (c + 3 == n - 1) ? C.w : cell(C.w, N.w, S.w, C.z, ev);
        }
        *reinterpret_cast<float4*>(out + (4u * rg + k) * kTile + 4u * q) = O;
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");    // smem writes -> TMA unit
      __syncthreads();
      if (tid == 0) {
        asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];"
                     :: "l"(reinterpret_cast<uint64_t>(&g.tma_out)), "r"(u32(out)), "r"(c0), "r"(r0) : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      }
    }
    if (tid == 0) *phase() = ph;     // every thread read it before the tile loop's barriers
  }
};

}  // namespace flep
