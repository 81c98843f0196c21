// bodies.cuh — original block bodies of the memory-bound workloads.
//
// Each body executes a contiguous range [b0, b1) of ORIGINAL block indices with all threads of
// the CTA (the wrapper passes a chunk, the unwrapped twin passes one block). Per-block work is
// identical in both, so wrapped, unwrapped, sliced and preempted-then-resumed runs produce
// bit-identical outputs (SURVEY §8(c) "Parity criteria").
//
//   SAXPY  (VA-shaped, Table 1): block b = elements [256b, 256b+256); 128-bit ld/st.
//   SpMV   (SPMV): block b = rows [128b, 128b+128); CSR-stream, fixed-order row sums (a
//          CSR-vector form with 4 lanes per row is FLEP_SPMV_VECTOR=1).
//   Stencil5 (BJ "2D stencil"; PF/CFD-shaped): block (tx, ty) = 64x64 output tile; each thread
//          produces a 4x4 patch with 128-bit loads; halo rows/columns come from L1/L2.
#pragma once
#include <cstdint>
#include "../../include/flep.h"
#include "flep_device.cuh"

#ifndef FLEP_SPMV_U
#define FLEP_SPMV_U 4
#endif
#ifndef FLEP_SPMV_VECTOR
#define FLEP_SPMV_VECTOR 0           // 0: CSR-stream body (products staged in shared memory);
                                     // 1: CSR-vector body (4 lanes per row, shuffle reduction)
#endif
#ifndef FLEP_SPMV_ASYNC
#define FLEP_SPMV_ASYNC 0            // 1: CSR-stream body whose col/val tiles arrive by cp.async
#endif
#ifndef FLEP_SPMV_AU
#define FLEP_SPMV_AU 8               // gathers in flight per thread in the cp.async body
#endif
#ifndef FLEP_SPMV_MINB
#define FLEP_SPMV_MINB 8             // SpMV CSR-stream: __launch_bounds__ min blocks (8 -> 32 registers)
#endif
#ifndef FLEP_SPMV_TILE
#define FLEP_SPMV_TILE 2048          // SpMV CSR-stream: nonzeros per shared-memory product tile
#endif
#ifndef FLEP_SPMV_ROWS
#define FLEP_SPMV_ROWS 128           // rows per original block (flep.py SPMV_ROWS_PER_BLOCK)
#endif

namespace flep {

__device__ __forceinline__ int4 ldcs4(const int4* p) { return __ldcs(p); }
__device__ __forceinline__ void stcs4(int4* p, int4 v) { __stcs(p, v); }

// ---------------------------------------------------------------------------------------------
// SAXPY: y <- a*x + y. int32 wraps modulo 2^32 (computed in uint32); fp32 uses one fma per element.
template <bool kInt>
struct SaxpyBody : NoResources {
  static constexpr int kThreads = 256;
  static constexpr int kMinBlocks = 8;
  static constexpr uint32_t kBlockElems = 256;
  using Args = typename std::conditional<kInt, flep_saxpy_i32_args, flep_saxpy_f32_args>::type;

  __device__ __forceinline__ static uint32_t op(uint32_t a, uint32_t x, uint32_t y, std::true_type) {
    return a * x + y;
  }
  __device__ __forceinline__ static uint32_t op(uint32_t a, uint32_t x, uint32_t y, std::false_type) {
    return __float_as_uint(fmaf(__uint_as_float(a), __uint_as_float(x), __uint_as_float(y)));
  }
  __device__ __forceinline__ static uint32_t f(uint32_t a, uint32_t x, uint32_t y) {
    return op(a, x, y, std::integral_constant<bool, kInt>{});
  }

  __device__ static void run(const Args& g, uint32_t b0, uint32_t b1, uint32_t, uint32_t) {
    const uint64_t e0 = (uint64_t)b0 * kBlockElems;
    const uint64_t e1 = min((uint64_t)b1 * kBlockElems, (uint64_t)g.n);
    if (e0 >= e1) return;
    const uint32_t a = kInt ? (uint32_t)g.a : __float_as_uint((float)g.a);
    const uint32_t* __restrict__ x = reinterpret_cast<const uint32_t*>(g.x) + e0;
    uint32_t* __restrict__ y = reinterpret_cast<uint32_t*>(g.y) + e0;
    const uint32_t nvec = (uint32_t)((e1 - e0) >> 2);
    const int4* __restrict__ x4 = reinterpret_cast<const int4*>(x);
    int4* __restrict__ y4 = reinterpret_cast<int4*>(y);
    constexpr uint32_t U = 2;                    // 2 x 128-bit loads of x and of y in flight
    uint32_t v = threadIdx.x;
    for (; v + (U - 1) * kThreads < nvec; v += U * kThreads) {
      int4 xv[U], yv[U];
#pragma unroll
      for (uint32_t u = 0; u < U; ++u) { xv[u] = ldcs4(x4 + v + u * kThreads); yv[u] = ldcs4(y4 + v + u * kThreads); }
#pragma unroll
      for (uint32_t u = 0; u < U; ++u) {
        int4 r;
        r.x = (int)f(a, (uint32_t)xv[u].x, (uint32_t)yv[u].x);
        r.y = (int)f(a, (uint32_t)xv[u].y, (uint32_t)yv[u].y);
        r.z = (int)f(a, (uint32_t)xv[u].z, (uint32_t)yv[u].z);
        r.w = (int)f(a, (uint32_t)xv[u].w, (uint32_t)yv[u].w);
        stcs4(y4 + v + u * kThreads, r);
      }
    }
    for (; v < nvec; v += kThreads) {
      const int4 xv = ldcs4(x4 + v), yv = ldcs4(y4 + v);
      int4 r;
      r.x = (int)f(a, (uint32_t)xv.x, (uint32_t)yv.x);
      r.y = (int)f(a, (uint32_t)xv.y, (uint32_t)yv.y);
      r.z = (int)f(a, (uint32_t)xv.z, (uint32_t)yv.z);
      r.w = (int)f(a, (uint32_t)xv.w, (uint32_t)yv.w);
      stcs4(y4 + v, r);
    }
    const uint64_t tail = e0 + ((uint64_t)nvec << 2);   // ragged tail (n % 4 != 0)
    for (uint64_t e = tail + threadIdx.x; e < e1; e += kThreads) y[e - e0] = f(a, x[e - e0], y[e - e0]);
  }
};

// ---------------------------------------------------------------------------------------------
// SpMV-CSR fp32: y[r] = sum_p val[p] * x[col[p]]. Block b = rows [128b, 128b+128).
// Default: the CSR-stream form. The CSR-vector form (FLEP_SPMV_VECTOR=1) is 4 % faster unwrapped
// and 2.5 % as the C = 1 worker (profiles/r01_spmv_vector.jsonl) but its warps finish a block at
// more spread-out times (rows of different lengths per warp), which lengthened the victim's
// drain from 9.1 to 10.2 us p50 (r01_bench_spmv_vector.json): latency wins here. CSR-stream: the rowptr slice of up to 256 rows (two blocks of a chunk; one block in the
// unwrapped kernel) goes to smem; all 256 threads then stream the rows' contiguous nnz range in
// tiles of kTile entries (coalesced col/val loads, independent x gathers, U in flight per thread),
// writing products to smem; thread t sums row r0+t's products in ascending p order. Per-row
// summation order does not depend on the grouping, so every execution of a block (wrapped,
// unwrapped, preempted and resumed) gives bit-identical results.
struct SpmvBody : NoResources {
  static constexpr int kThreads = 256;
  static constexpr int kMinBlocks = FLEP_SPMV_MINB;   // resident CTAs per SM the register budget is sized for
  static constexpr uint32_t kRowsPerBlock = FLEP_SPMV_ROWS;
  static constexpr uint32_t kTile = FLEP_SPMV_TILE;     // products staged per tile (smem)
  using Args = flep_spmv_args;

  static constexpr uint32_t kGroupRows = 256;     // rows streamed together (2 blocks of a chunk)

#if FLEP_SPMV_VECTOR
  // CSR-vector form: 4 lanes per row (8 rows per warp, 64 rows per CTA pass); lane l of a row's
  // group takes the row's nonzeros p = s+l, s+l+4, ... in ascending order (U in flight), and the
  // group's 4 partial sums are combined by two butterfly shuffles (every lane ends with the same
  // bits). No shared memory and no CTA barrier; the order is fixed, so wrapped, unwrapped and
  // resumed runs stay bit-identical.
  __device__ static void run(const Args& g, uint32_t b0, uint32_t b1, uint32_t, uint32_t) {
    constexpr int U = FLEP_SPMV_U;
    const uint32_t tid = threadIdx.x;
    const int32_t sub = (int32_t)(tid & 3u);
    const uint32_t row_end = min(b1 * kRowsPerBlock, g.rows);
    for (uint32_t r0 = b0 * kRowsPerBlock; r0 < row_end; r0 += kThreads / 4) {
      const uint32_t r = r0 + (tid >> 2);
      const bool valid = r < row_end;
      const int32_t s = valid ? __ldg(g.rowptr + r) : 0, e = valid ? __ldg(g.rowptr + r + 1) : 0;
      float acc = 0.f;
      for (int32_t p = s + sub; p < e; p += 4 * U) {
        int32_t c[U];
        float v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int32_t q = p + 4 * u;
          c[u] = q < e ? __ldcs(g.col + q) : 0;
          v[u] = q < e ? __ldcs(g.val + q) : 0.f;
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const float xv = __ldg(g.x + c[u]);
          if (p + 4 * u < e) acc += v[u] * xv;
        }
      }
      acc += __shfl_xor_sync(0xffffffffu, acc, 1);
      acc += __shfl_xor_sync(0xffffffffu, acc, 2);
      if (valid && sub == 0) __stcs(g.y + r, acc);
    }
  }
#elif FLEP_SPMV_ASYNC
  // CSR-stream with the tile's col/val staged by cp.async (16-B copies, no registers held while
  // they are in flight): one HBM round trip per tile, then every gather of the tile in flight
  // (U = FLEP_SPMV_AU per thread, indices read from shared memory). Products are formed in place
  // (val * x, the same fp32 multiply) and summed per row in ascending p, as in the form below, so
  // results stay bit-identical to it.
  __device__ static void cp_async16(void* dst, const void* src) {
    const uint32_t d = static_cast<uint32_t>(__cvta_generic_to_shared(dst));
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(d), "l"(src) : "memory");
  }
  __device__ static void run(const Args& g, uint32_t b0, uint32_t b1, uint32_t, uint32_t) {
    __shared__ int32_t s_rp[kGroupRows + 1];
    __shared__ __align__(16) int32_t s_col[kTile + 4];
    __shared__ __align__(16) float s_val[kTile + 4];
    const uint32_t tid = threadIdx.x;
    const uint32_t row_end = min(b1 * kRowsPerBlock, g.rows);
    for (uint32_t r0 = b0 * kRowsPerBlock; r0 < row_end; r0 += kGroupRows) {
      const uint32_t nr = min(kGroupRows, row_end - r0);
      if (tid <= nr) s_rp[tid] = __ldg(g.rowptr + r0 + tid);
      if (tid == 0 && nr == kGroupRows) s_rp[kGroupRows] = __ldg(g.rowptr + r0 + kGroupRows);
      body_sync<kThreads>();
      const int32_t p0 = s_rp[0], p1 = s_rp[nr];
      int32_t my_s = 0, my_e = 0;
      if (tid < nr) { my_s = s_rp[tid]; my_e = s_rp[tid + 1]; }
      // An all-empty group runs no tile (whose barriers order these s_rp reads before the next
      // group's s_rp writes): order them here. p0/p1 are the same in every thread (uniform).
      if (p0 >= p1) body_sync<kThreads>();
      float acc = 0.f;
      for (int32_t base = p0; base < p1; base += (int32_t)kTile) {
        const int32_t n = min((int32_t)kTile, p1 - base);
        const int32_t a0 = base & ~3;                 // 16-B aligned (elements before base exist)
        const int32_t off = base - a0;
        const int32_t a1 = (base + n) & ~3;           // aligned end: never past the arrays
        for (int32_t j = (int32_t)tid; 4 * j < a1 - a0; j += kThreads) {
          cp_async16(&s_col[4 * j], g.col + a0 + 4 * j);
          cp_async16(&s_val[4 * j], g.val + a0 + 4 * j);
        }
        const int32_t t0 = max(a1, base);             // < 4 tail elements by plain loads
        if ((int32_t)tid < base + n - t0) {
          s_col[t0 - a0 + (int32_t)tid] = __ldcs(g.col + t0 + tid);
          s_val[t0 - a0 + (int32_t)tid] = __ldcs(g.val + t0 + tid);
        }
        asm volatile("cp.async.wait_all;" ::: "memory");
        body_sync<kThreads>();
        constexpr int U = FLEP_SPMV_AU;
        for (int32_t i0 = (int32_t)tid; i0 < n; i0 += U * kThreads) {
          int32_t c[U];
          float xv[U];
#pragma unroll
          for (int u = 0; u < U; ++u) {
            const int32_t i = i0 + u * kThreads;
            c[u] = i < n ? s_col[off + i] : 0;
          }
#pragma unroll
          for (int u = 0; u < U; ++u) xv[u] = __ldg(g.x + c[u]);
#pragma unroll
          for (int u = 0; u < U; ++u) {
            const int32_t i = i0 + u * kThreads;
            if (i < n) s_val[off + i] = s_val[off + i] * xv[u];
          }
        }
        body_sync<kThreads>();
        if (tid < nr) {                        // row r0+tid: its products in ascending p order
          const int32_t lo = max(my_s, base), hi = min(my_e, base + n);
          for (int32_t p = lo; p < hi; ++p) acc += s_val[off + p - base];
        }
        body_sync<kThreads>();
      }
      if (tid < nr) __stcs(g.y + r0 + tid, acc);
    }
  }
#else
  __device__ static void run(const Args& g, uint32_t b0, uint32_t b1, uint32_t, uint32_t) {
    __shared__ int32_t s_rp[kGroupRows + 1];
    __shared__ float s_prod[kTile];
    const uint32_t tid = threadIdx.x;
    const uint32_t row_end = min(b1 * kRowsPerBlock, g.rows);
    for (uint32_t r0 = b0 * kRowsPerBlock; r0 < row_end; r0 += kGroupRows) {
      const uint32_t nr = min(kGroupRows, row_end - r0);
      if (tid <= nr) s_rp[tid] = __ldg(g.rowptr + r0 + tid);
      if (tid == 0 && nr == kGroupRows) s_rp[kGroupRows] = __ldg(g.rowptr + r0 + kGroupRows);
      body_sync<kThreads>();
      const int32_t p0 = s_rp[0], p1 = s_rp[nr];
      int32_t my_s = 0, my_e = 0;
      if (tid < nr) { my_s = s_rp[tid]; my_e = s_rp[tid + 1]; }
      // An all-empty group runs no tile (whose barriers order these s_rp reads before the next
      // group's s_rp writes): order them here. p0/p1 are the same in every thread (uniform).
      if (p0 >= p1) body_sync<kThreads>();
      float acc = 0.f;
      for (int32_t base = p0; base < p1; base += (int32_t)kTile) {
        const int32_t n = min((int32_t)kTile, p1 - base);
        constexpr int U = FLEP_SPMV_U;
        for (int32_t i0 = (int32_t)tid; i0 < n; i0 += U * kThreads) {
          int32_t c[U];
          float v[U], xv[U];
#pragma unroll
          for (int u = 0; u < U; ++u) {
            const int32_t i = i0 + u * kThreads;
            c[u] = i < n ? __ldcs(g.col + base + i) : 0;
            v[u] = i < n ? __ldcs(g.val + base + i) : 0.f;
          }
#pragma unroll
          for (int u = 0; u < U; ++u) xv[u] = __ldg(g.x + c[u]);
#pragma unroll
          for (int u = 0; u < U; ++u) {
            const int32_t i = i0 + u * kThreads;
            if (i < n) s_prod[i] = v[u] * xv[u];
          }
        }
        body_sync<kThreads>();
        if (tid < nr) {                        // row r0+tid: its products in ascending p order
          const int32_t lo = max(my_s, base), hi = min(my_e, base + n);
          for (int32_t p = lo; p < hi; ++p) acc += s_prod[p - base];
        }
        body_sync<kThreads>();
      }
      if (tid < nr) __stcs(g.y + r0 + tid, acc);
    }
  }
#endif
};

// ---------------------------------------------------------------------------------------------
// 5-point stencil, out-of-place. Interior: fp32 0.5*c + 0.125*(n + s + w + e); int32
// 4c - n - s - w - e (mod 2^32). Boundary rows/columns copied through.
template <bool kInt>
struct Stencil5Body : NoResources {
  static constexpr int kThreads = 256;
  static constexpr int kMinBlocks = 4;
  static constexpr uint32_t kTile = 64;
  using Args = flep_stencil_args;

  __device__ __forceinline__ static uint32_t cell(uint32_t c, uint32_t n, uint32_t s, uint32_t w, uint32_t e) {
    if (kInt) return 4u * c - n - s - w - e;
    const float fc = __uint_as_float(c), fn = __uint_as_float(n), fs = __uint_as_float(s),
                fw = __uint_as_float(w), fe = __uint_as_float(e);
    return __float_as_uint(0.5f * fc + 0.125f * (((fn + fs) + fw) + fe));
  }

  // Vector path (n % 4 == 0): thread (q, rg) owns columns [c0+4q, c0+4q+4) of rows
  // r0+4rg .. r0+4rg+3. It loads the 6 rows r-1..r+4 of its 4-column strip (128-bit) and the
  // west/east neighbours of its 4 rows up front (14 independent loads in flight), then computes.
  // Thread tid's work depends on (b, tid) only, so warp w of a block (threads 32w..32w+31, rows
  // r0+8w..r0+8w+7) is an independent task of the warp-task worker (R30).
  static constexpr uint32_t kWarpTasks = kThreads / 32;
  __device__ __forceinline__ static void run_thread(const Args& g, uint32_t b, uint32_t tid, uint32_t gx) {
    const uint32_t n = g.n;
    const uint32_t* __restrict__ in = reinterpret_cast<const uint32_t*>(g.in);
    uint32_t* __restrict__ out = reinterpret_cast<uint32_t*>(g.out);
    const uint32_t tx = b % gx, ty = b / gx;
    const uint32_t r0 = ty * kTile, c0 = tx * kTile;
    if ((n & 3u) == 0) {
      const uint32_t q = tid & 15u, rg = tid >> 4;   // 16 strips x 16 row groups
      const uint32_t c = c0 + 4u * q;
      const uint32_t rb = r0 + 4u * rg;
      if (c >= n || rb >= n) return;
      uint4 R[6];
      uint32_t Wv[4], Ev[4];
#pragma unroll
      for (int i = 0; i < 6; ++i) {
        const int32_t r = (int32_t)rb - 1 + i;
        R[i] = (r >= 0 && r < (int32_t)n) ? __ldg(reinterpret_cast<const uint4*>(in + (size_t)r * n + c))
                                          : make_uint4(0, 0, 0, 0);
      }
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const uint32_t r = rb + i;
        Wv[i] = (r < n && c > 0) ? __ldg(in + (size_t)r * n + c - 1) : 0u;
        Ev[i] = (r < n && c + 4 < n) ? __ldg(in + (size_t)r * n + c + 4) : 0u;
      }
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const uint32_t r = rb + i;
        if (r >= n) break;
        const uint4 C = R[i + 1], N = R[i], S = R[i + 2];
        uint4 O;
        if (r == 0 || r == n - 1) {
          O = C;
        } else {
          O.x = (c == 0) ? C.x : cell(C.x, N.x, S.x, Wv[i], C.y);
          O.y = cell(C.y, N.y, S.y, C.x, C.z);
          O.z = cell(C.z, N.z, S.z, C.y, C.w);
          O.w = (c + 3 == n - 1) ? C.w : cell(C.w, N.w, S.w, C.z, Ev[i]);
        }
        __stcs(reinterpret_cast<uint4*>(out + (size_t)r * n + c), O);
      }
    } else {
      // scalar path for n % 4 != 0 (ragged rows)
      for (uint32_t t = tid; t < kTile * kTile; t += kThreads) {
        const uint32_t r = r0 + t / kTile, c = c0 + t % kTile;
        if (r >= n || c >= n) continue;
        const size_t off = (size_t)r * n + c;
        const uint32_t C = __ldg(in + off);
        if (r == 0 || r == n - 1 || c == 0 || c == n - 1) { out[off] = C; continue; }
        out[off] = cell(C, __ldg(in + off - n), __ldg(in + off + n), __ldg(in + off - 1), __ldg(in + off + 1));
      }
    }
  }
  __device__ static void run(const Args& g, uint32_t b0, uint32_t b1, uint32_t gx, uint32_t) {
    for (uint32_t b = b0; b < b1; ++b) run_thread(g, b, threadIdx.x, gx);
  }
  __device__ static void run_warp(const Args& g, uint32_t task, uint32_t gx, uint32_t) {
    run_thread(g, task / kWarpTasks, (task % kWarpTasks) * 32u + (threadIdx.x & 31u), gx);
  }
};

// ---------------------------------------------------------------------------------------------
// SpMV-CSR fp32, CSR-vector form (FLEP_BODY_SPMV_CSR_F32_VEC): block b = rows [128b, 128b+128),
// 4 lanes per row, 8 rows per warp per pass, 2 passes: warp w of block b owns rows
// 128b + 64*pass + 8w + lane/4. Lane l of a row's group sums the row's nonzeros p = s+l, s+l+4,
// ... in ascending order (U in flight) and the group's 4 partial sums are combined by two
// butterfly shuffles. No shared memory and no CTA barrier: warp w's rows are an independent task
// of the warp-task worker (R30); every execution of a row is the same arithmetic in the same order.
struct SpmvVecBody : NoResources {
  static constexpr int kThreads = 256;
  static constexpr int kMinBlocks = 8;
  static constexpr uint32_t kRowsPerBlock = 128;
  static constexpr uint32_t kWarpTasks = kThreads / 32;
  using Args = flep_spmv_args;

  __device__ __forceinline__ static void rows_of_warp(const Args& g, uint32_t b, uint32_t w, uint32_t lane) {
    constexpr int U = FLEP_SPMV_U;
    const int32_t sub = (int32_t)(lane & 3u);
#pragma unroll 1
    for (uint32_t pass = 0; pass < 2; ++pass) {
      const uint32_t r = b * kRowsPerBlock + pass * 64u + w * 8u + (lane >> 2);
      const bool valid = r < g.rows;
      const int32_t s = valid ? __ldg(g.rowptr + r) : 0, e = valid ? __ldg(g.rowptr + r + 1) : 0;
      float acc = 0.f;
      for (int32_t p = s + sub; p < e; p += 4 * U) {
        int32_t c[U];
        float v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int32_t q = p + 4 * u;
          c[u] = q < e ? __ldcs(g.col + q) : 0;
          v[u] = q < e ? __ldcs(g.val + q) : 0.f;
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const float xv = __ldg(g.x + c[u]);
          if (p + 4 * u < e) acc += v[u] * xv;
        }
      }
      acc += __shfl_xor_sync(0xffffffffu, acc, 1);
      acc += __shfl_xor_sync(0xffffffffu, acc, 2);
      if (valid && sub == 0) __stcs(g.y + r, acc);
    }
  }
  __device__ static void run(const Args& g, uint32_t b0, uint32_t b1, uint32_t, uint32_t) {
    for (uint32_t b = b0; b < b1; ++b) rows_of_warp(g, b, threadIdx.x >> 5, threadIdx.x & 31u);
  }
  __device__ static void run_warp(const Args& g, uint32_t task, uint32_t, uint32_t) {
    rows_of_warp(g, task / kWarpTasks, task % kWarpTasks, threadIdx.x & 31u);
  }
};

}  // namespace flep
