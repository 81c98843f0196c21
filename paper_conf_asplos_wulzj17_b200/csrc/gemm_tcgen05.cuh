// gemm_tcgen05.cuh — the dense-contraction body (MM, Table 1): C = A·Bᵀ with A
// [M,K] and B [N,K] bf16 row-major (K-major "TN"), fp32 accumulation in TMEM, bf16 output.
//
// One original block = one 128x256 output tile. Inside the FLEP worker the CTA is warp-
// specialised (sm_100a):
//   warp 0 lane 0 : TMA producer — 128x64 A box + 256x64 B box per k-step, SWIZZLE_128B, into a
//                   4-stage smem ring (full/empty mbarriers)
//   warp 1 lane 0 : MMA issuer — tcgen05.mma.cta_group::1.kind::f16, M=128 N=256 K=16, four per
//                   k-step, accumulator in TMEM (256 columns); tcgen05.commit frees smem stages
//                   and finally signals the epilogue
//   warp 2        : TMEM allocator (setup) / deallocator (teardown: before any exit, a7)
//   warps 4..7    : epilogue — tcgen05.ld 32x32b.x32 → bf16 → global, then release the
//                   accumulator (tmem_empty)
// Pipeline phases persist in shared memory across chunks, so a worker's consecutive tasks share
// one pipeline; the wrapper's barrier separates chunks (the poll point).
//
// In-tile preemption (kernels registered with FLEP_KFLAG_IN_TILE): the producer also
// polls the control word every kInTilePoll k-steps inside a tile. On a request naming its SM it
// stops issuing k-steps and sends a stop marker through the stage ring; the MMA thread commits
// the partial accumulator, the epilogue spills it (fp32, exact) to the worker's slot and the
// producer records {tile, next k-step, chunk end}. Worker i of the next epoch restores the
// accumulator into TMEM (tcgen05.st) and continues the same k-loop: every k-step of every tile is
// accumulated exactly once, in the same order, so the result is bit-identical to an
// uninterrupted run. Preemption latency drops from one tile (~55 us at 8192^3) to a few k-steps.
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <cstdint>

#include "../../include/flep.h"
#include "flep_device.cuh"

#ifndef FLEP_GEMM_GROUP
#define FLEP_GEMM_GROUP 16
#endif
#ifndef FLEP_GEMM_KPOLL
#define FLEP_GEMM_KPOLL 4         // k-steps (BK = 64 each) between in-tile polls (sweep: 2 -> 7.4 us drain, +0.4 %; 4 -> 8.7 us, +0.1 %; 8 -> 11.9 us, +0.5 %)
#endif

namespace flep {

struct GemmArgsDev {
  CUtensorMap tma_a;           // A [M,K] bf16, box {64, 128}, SWIZZLE_128B
  CUtensorMap tma_b;           // B [N,K] bf16, box {64, 256}, SWIZZLE_128B
  CUtensorMap tma_c;           // C [M,N] bf16, box {64, 32}, SWIZZLE_128B (epilogue bulk stores)
  __nv_bfloat16* c;            // C [M,N] bf16 row-major
  uint32_t m, n, k;
};

struct GemmBody {
  static constexpr int kThreads = 256;
  static constexpr int kMinBlocks = 1;
  static constexpr uint32_t BM = 128, BN = 256, BK = 64, UMMA_K = 16, STAGES = 4;
  static constexpr uint32_t kBytesA = BM * BK * 2, kBytesB = BN * BK * 2, kStage = kBytesA + kBytesB;
  static constexpr uint32_t kTmemCols = 512;           // two 128x256 fp32 accumulators
  static constexpr uint32_t QDEPTH = 4;                // tile queue: scheduler -> MMA / epilogue
  // epilogue staging after the state block: per epilogue warp two 4 KB buffers (32 rows x 64
  // bf16 columns, SWIZZLE_128B) written to C by bulk tensor stores (store_bulk)
  static constexpr uint32_t kEpiBuf = 32 * 128;
  static constexpr size_t kDynSmem = 1024 + STAGES * kStage + 1024 + 4 * 2 * kEpiBuf;
  static_assert(kDynSmem <= 232448, "shared memory per block");
  static constexpr bool kPersistent = true;
  using Args = GemmArgsDev;

  struct State {                      // lives after the stage ring
    uint64_t full[STAGES], empty[STAGES], tmem_full, tmem_empty;
    uint64_t tfull[2], tempty[2];     // persistent loop: double-buffered accumulators
    uint64_t qfull[QDEPTH], qempty[QDEPTH];
    uint64_t trest[2];                // epilogue restored a spilled accumulator into this half
    uint32_t tile_q[QDEPTH];
    uint32_t tile_kb0[QDEPTH];        // first k-step of the tile (> 0: continue a spilled tile)
    uint32_t stage_stop[STAGES];      // 1: this stage is a stop marker (no data): written by the
                                      // producer after the stage's empty wait, read by the MMA
                                      // after its full wait, so the ring orders every access
    uint32_t acc_kend[2];             // MMA -> epilogue: k-steps accumulated in this half
    uint32_t tmem_base;
    uint32_t p_stage, p_phase;        // producer
    uint32_t m_stage, m_phase, m_acc; // MMA issuer
    uint32_t e_acc[4];                // epilogue, one copy per epilogue warp (no cross-warp WAR)
  };

  __device__ static uint8_t* ring() {
    extern __shared__ uint8_t dsmem[];
    const uint32_t a = static_cast<uint32_t>(__cvta_generic_to_shared(dsmem));
    return dsmem + (((a + 1023u) & ~1023u) - a);
  }
  __device__ static State* state() { return reinterpret_cast<State*>(ring() + STAGES * kStage); }
  __device__ static uint32_t smem_u32(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }
  __device__ static uint8_t* epi_buf(uint32_t q) { return ring() + STAGES * kStage + 1024 + 2 * q * kEpiBuf; }

  __device__ static void mbar_init(uint64_t* b, uint32_t n) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(b)), "r"(n) : "memory");
  }
  __device__ static void mbar_wait(uint64_t* b, uint32_t parity) {
    asm volatile(
        "{\n .reg .pred p;\n W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        " @!p bra W;\n}\n" :: "r"(smem_u32(b)), "r"(parity) : "memory");
  }
  __device__ static void mbar_arrive(uint64_t* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(b)) : "memory");
  }
  __device__ static void mbar_expect_tx(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(b)), "r"(bytes) : "memory");
  }
  __device__ static void tma_2d(const CUtensorMap* map, void* dst, uint64_t* bar, int32_t x, int32_t y) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
        :: "r"(smem_u32(dst)), "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(x), "r"(y)
        : "memory");
  }
  // Original block b -> output tile (tm, tn). Blocks are numbered in bands of GROUP tile-rows,
  // column by column inside a band, so the tiles that run concurrently share B panels in L2.
  static constexpr uint32_t GROUP = FLEP_GEMM_GROUP;
  __device__ static uint32_t p_gy(const Args& g) { return g.m / BM; }
  __device__ static void tile_coords(uint32_t b, uint32_t gx, uint32_t gy, int32_t& tm, int32_t& tn) {
    const uint32_t band = GROUP * gx;
    const uint32_t grp = b / band, r = b % band;
    const uint32_t rows = min(GROUP, gy - grp * GROUP);
    tm = (int32_t)(grp * GROUP + r % rows);
    tn = (int32_t)(r / rows);
  }
  // K-major, SWIZZLE_128B smem matrix descriptor (sm_100 UMMA): start>>4, LBO 16 B (unused for
  // swizzled K-major), SBO 1024 B (8 rows x 128 B), version 1, layout SWIZZLE_128B (2).
  __device__ static uint64_t sdesc(uint32_t saddr) {
    return (uint64_t)((saddr >> 4) & 0x3FFFu) | ((uint64_t)1u << 16) | ((uint64_t)(1024u >> 4) << 32) |
           ((uint64_t)1u << 46) | ((uint64_t)2u << 61);
  }
  // kind::f16 instruction descriptor: D f32, A/B bf16, both K-major, N = 256, M = 128.
  static constexpr uint32_t kIdesc = (1u << 4) | (1u << 7) | (1u << 10) | ((BN >> 3) << 17) | ((BM >> 4) << 24);

  __device__ static void setup(const Args&) {
    State* s = state();
    const uint32_t warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) {
      for (uint32_t i = 0; i < STAGES; ++i) { mbar_init(&s->full[i], 1); mbar_init(&s->empty[i], 1); }
      mbar_init(&s->tmem_full, 1);
      mbar_init(&s->tmem_empty, 128);
      // tfull: the MMA's tcgen05.commit + a plain arrive of the MMA thread (publishes acc_kend)
      for (uint32_t i = 0; i < 2; ++i) {
        mbar_init(&s->tfull[i], 2); mbar_init(&s->tempty[i], 128); mbar_init(&s->trest[i], 128);
      }
      for (uint32_t i = 0; i < QDEPTH; ++i) { mbar_init(&s->qfull[i], 1); mbar_init(&s->qempty[i], 5); }
      s->p_stage = s->p_phase = s->m_stage = s->m_phase = s->m_acc = 0;
      s->e_acc[0] = s->e_acc[1] = s->e_acc[2] = s->e_acc[3] = 0;
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 2) {
      asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                   :: "r"(smem_u32(&s->tmem_base)), "r"(kTmemCols) : "memory");
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  }

  __device__ static void teardown(const Args&) {
    State* s = state();
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if ((threadIdx.x >> 5) == 2)
      asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(s->tmem_base), "r"(kTmemCols) : "memory");
  }

  __device__ static void run(const Args& g, uint32_t b0, uint32_t b1, uint32_t gx, uint32_t) {
    State* s = state();
    uint8_t* base = ring();
    const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31u;
    const uint32_t nk = g.k / BK;
    if (warp == 0) {
      if (lane == 0) {                                     // ---- TMA producer
        uint32_t st = s->p_stage, ph = s->p_phase;
        for (uint32_t b = b0; b < b1; ++b) {
          int32_t tm, tn;
          tile_coords(b, gx, p_gy(g), tm, tn);
          for (uint32_t kb = 0; kb < nk; ++kb) {
            mbar_wait(&s->empty[st], ph ^ 1u);
            uint8_t* sa = base + st * kStage;
            uint8_t* sb = sa + kBytesA;
            mbar_expect_tx(&s->full[st], kStage);
            tma_2d(&g.tma_a, sa, &s->full[st], (int32_t)(kb * BK), tm * (int32_t)BM);
            tma_2d(&g.tma_b, sb, &s->full[st], (int32_t)(kb * BK), tn * (int32_t)BN);
            if (++st == STAGES) { st = 0; ph ^= 1u; }
          }
        }
        s->p_stage = st; s->p_phase = ph;
      }
    } else if (warp == 1) {
      if (lane == 0) {                                     // ---- MMA issuer (one thread)
        uint32_t st = s->m_stage, ph = s->m_phase, acc = s->m_acc;
        const uint32_t tmem = s->tmem_base;
        for (uint32_t b = b0; b < b1; ++b) {
          mbar_wait(&s->tmem_empty, acc ^ 1u);             // epilogue drained the accumulator
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          for (uint32_t kb = 0; kb < nk; ++kb) {
            mbar_wait(&s->full[st], ph);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            const uint32_t sa = smem_u32(base + st * kStage), sb = sa + kBytesA;
#pragma unroll
            for (uint32_t k = 0; k < BK / UMMA_K; ++k) {
              const uint64_t da = sdesc(sa + k * UMMA_K * 2), db = sdesc(sb + k * UMMA_K * 2);
              const uint32_t accum = (kb | k) ? 1u : 0u;
              asm volatile(
                  "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
                  " tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n"
                  :: "r"(tmem), "l"(da), "l"(db), "r"(kIdesc), "r"(accum) : "memory");
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                         :: "r"(smem_u32(&s->empty[st])) : "memory");
            if (++st == STAGES) { st = 0; ph ^= 1u; }
          }
          asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                       :: "r"(smem_u32(&s->tmem_full)) : "memory");
          acc ^= 1u;
        }
        s->m_stage = st; s->m_phase = ph; s->m_acc = acc;
      }
    } else if (warp >= 4) {                                // ---- epilogue (128 threads)
      const uint32_t q = warp - 4;                         // TMEM lanes [32q, 32q+32)
      uint32_t acc = s->e_acc[q], it = 0;
      const uint32_t tmem = s->tmem_base + ((q * 32u) << 16);
      for (uint32_t b = b0; b < b1; ++b) {
        int32_t tm, tn;
        tile_coords(b, gx, p_gy(g), tm, tn);
        mbar_wait(&s->tmem_full, acc);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        store_bulk(&g.tma_c, epi_buf(q), tmem, 0, BN, tn * (int32_t)BN, tm * (int32_t)BM + (int32_t)(q * 32u), lane, it);
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        mbar_arrive(&s->tmem_empty);
        acc ^= 1u;
      }
      bulk_wait_all(lane);
      if (lane == 0) s->e_acc[q] = acc;
    }
  }

  static constexpr uint32_t kInTilePoll = FLEP_GEMM_KPOLL;
  static constexpr uint32_t kMinLeft = 4;      // closer than this to the tile's end: finish it

  __device__ static float4* spill_slot(const WorkerParams& p) {
    return reinterpret_cast<float4*>(reinterpret_cast<uint8_t*>(p.partial) + partial_header_bytes(p.workers) +
                                     (size_t)blockIdx.x * kSpillBytes);
  }
  // TMEM <-> registers, 32 lanes x 32 columns per warp
  __device__ static void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
  }
  __device__ static void tmem_st32(uint32_t taddr, const uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
        "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};"
        :: "r"(taddr), "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]),
           "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]),
           "r"(r[16]), "r"(r[17]), "r"(r[18]), "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]),
           "r"(r[24]), "r"(r[25]), "r"(r[26]), "r"(r[27]), "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31])
        : "memory");
  }

  // Epilogue store of one warp's 32 accumulator rows (TMEM lanes of tmem_w), columns
  // [c_begin, c_end) in steps of 64: TMEM -> bf16 -> one of the warp's two staging buffers (row =
  // lane, 16-B chunk c at c ^ (lane & 7): the SWIZZLE_128B layout of the C tensor map) -> one bulk
  // tensor store of 32 x 64 issued by lane 0 at (x0 + c, y0), so the store of one chunk overlaps
  // the next chunk's TMEM loads and C is written in full 128-B lines (the per-lane row stores it
  // replaces issued one 16-B request per row). `it` counts the warp's stores (buffer it & 1);
  // the warp ends with bulk_wait_all() before the CTA can exit. Used by both GEMM bodies.
  __device__ static void store_bulk(const CUtensorMap* tmc, uint8_t* bufs, uint32_t tmem_w, uint32_t c_begin,
                                    uint32_t c_end, int32_t x0, int32_t y0, uint32_t lane, uint32_t& it) {
#pragma unroll 1
    for (uint32_t c0 = c_begin; c0 < c_end; c0 += 64) {
      uint32_t o[32];
#pragma unroll
      for (uint32_t hh = 0; hh < 2; ++hh) {
        uint32_t v[32];
        tmem_ld32(tmem_w + c0 + 32 * hh, v);
#pragma unroll
        for (int i = 0; i < 16; ++i) {
          __nv_bfloat162 hv = __floats2bfloat162_rn(__uint_as_float(v[2 * i]), __uint_as_float(v[2 * i + 1]));
          o[16 * hh + i] = *reinterpret_cast<uint32_t*>(&hv);
        }
      }
      if (it >= 2) {                                   // the store that used this buffer has read it
        if (lane == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
        __syncwarp();
      }
      uint8_t* buf = bufs + (it & 1u) * kEpiBuf;
      const uint32_t rowb = smem_u32(buf) + lane * 128u;
#pragma unroll
      for (uint32_t c = 0; c < 8; ++c)
        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};"
                     :: "r"(rowb + ((c ^ (lane & 7u)) << 4)), "r"(o[4 * c]), "r"(o[4 * c + 1]), "r"(o[4 * c + 2]),
                        "r"(o[4 * c + 3]) : "memory");
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // visible to the bulk store
      __syncwarp();
      if (lane == 0) {
        asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];"
                     :: "l"(reinterpret_cast<uint64_t>(tmc)), "r"(smem_u32(buf)), "r"(x0 + (int32_t)c0), "r"(y0)
                     : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      }
      ++it;
    }
  }
  __device__ static void bulk_wait_all(uint32_t lane) {    // this warp's bulk stores are complete
    if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    __syncwarp();
  }

  // ---- persistent FLEP worker loop (warp-specialised; chunk boundaries do not drain the
  // pipeline). tid 0 is the scheduler AND the TMA producer: it runs the FLEP scheduling step
  // (poll / fetch / trigger, next_chunk), pushes every tile of the fetched chunk into a 4-deep
  // smem queue, then issues that tile's TMA loads; a STOP sentinel ends the loop. The MMA thread
  // and the 4 epilogue warps consume the queue; accumulators alternate between two TMEM halves
  // so tile t's epilogue overlaps tile t+1's MMAs. Every fetched tile is computed (A4) — with
  // in-tile preemption, possibly across epochs (spill / restore, see the file header).
  __device__ static void persistent(const Args& g, const WorkerParams& p, WorkerShared& ws) {
    State* s = state();
    uint8_t* base = ring();
    const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31u;
    const uint32_t nk = g.k / BK;
    const uint32_t gx = p.gx;
    const bool in_tile = p.partial != nullptr;
    constexpr uint32_t STOP = 0xffffffffu;
    if (warp == 0) {
      if (lane == 0) {                                     // ---- scheduler + TMA producer
        SchedState sch;
        uint32_t qi = 0, qph = 0, st = 0, ph = 0;
        PartialTile* mine = in_tile ? reinterpret_cast<PartialTile*>(p.partial) + blockIdx.x : nullptr;
        uint32_t rb0 = STOP, rb1 = 0, rkb = 0;             // a spilled tile to continue first
        if (in_tile) {
          if (p.epoch == p.gen_first) {
            mine->valid = 0;                               // no record survives from another launch
          } else {
            const PartialTile e = *mine;                   // written by the previous grid
            if (e.valid) {
              sch.first = false;                           // (the launch is not complete)
              const uint32_t c = poll_ctrl(p);   // entry check (a2) before taking it
              if (should_yield(c, p, smid_reg())) {
                ws.reason = kReasonYield;                  // the record stays for a later epoch
                ws.partial = e.b_end - e.b;                // blocks still unfinished (R23)
                rb0 = STOP; rb1 = 1;                       // (marker: leave at once)
              } else {
                rb0 = e.b; rb1 = e.b_end; rkb = e.kb;
                mine->valid = 0;
                ws.blocks += e.b_end - e.b;                // counted again when they complete
              }
            }
          }
        }
        bool leave = (rb0 == STOP && rb1 == 1);
        while (!leave) {
          uint32_t b0, b1, kbs = 0;
          bool restoring = false;
          if (rb0 != STOP) {
            b0 = rb0; b1 = rb1; kbs = rkb; restoring = true;
            rb0 = STOP;
          } else {
            b0 = next_chunk(p, sch, ws);
            if (b0 == STOP) break;
            b1 = min(b0 + p.chunk, p.n_blocks);
          }
          for (uint32_t b = b0; b < b1; ++b) {
            const bool cont = restoring && b == b0;        // continue a spilled tile
            const uint32_t kb0 = cont ? kbs : 0u;
            mbar_wait(&s->qempty[qi], qph ^ 1u);
            s->tile_q[qi] = b;
            s->tile_kb0[qi] = kb0;
            mbar_arrive(&s->qfull[qi]);
            if (++qi == QDEPTH) { qi = 0; qph ^= 1u; }
            // coverage log: a tile counts once, when its chunk is first handed out (the tiles of
            // a chunk stopped in-tile are counted at the stop, not again when restored)
            if (p.cov && !restoring) atomicAdd(&p.cov[b], 1u);
            int32_t tm, tn;
            tile_coords(b, gx, p_gy(g), tm, tn);
            uint32_t kb = kb0, pend = 0;
            bool pend_valid = false, stop = false;
            for (; kb < nk; ++kb) {
              if (in_tile) {                               // amortised in-tile poll, issued one
                const uint32_t j = kb - kb0;               // half period before it is consumed
                if (pend_valid && j % kInTilePoll == kInTilePoll / 2) {
                  pend_valid = false;
                  if (nk - kb > kMinLeft && should_yield(pend, p, smid_reg())) { stop = true; break; }
                }
                if (j % kInTilePoll == 0 && j > 0) { pend = poll_ctrl(p); pend_valid = true; }
              }
              mbar_wait(&s->empty[st], ph ^ 1u);
              s->stage_stop[st] = 0u;
              uint8_t* sa = base + st * kStage;
              uint8_t* sb = sa + kBytesA;
              mbar_expect_tx(&s->full[st], kStage);
              tma_2d(&g.tma_a, sa, &s->full[st], (int32_t)(kb * BK), tm * (int32_t)BM);
              tma_2d(&g.tma_b, sb, &s->full[st], (int32_t)(kb * BK), tn * (int32_t)BN);
              if (++st == STAGES) { st = 0; ph ^= 1u; }
            }
            if (stop) {
              // stop marker: the next stage carries no data; the MMA sees it and commits
              mbar_wait(&s->empty[st], ph ^ 1u);
              s->stage_stop[st] = 1u;
              mbar_arrive(&s->full[st]);
              if (++st == STAGES) { st = 0; ph ^= 1u; }
              mine->b = b; mine->kb = kb; mine->b_end = b1; mine->valid = 1;
              if (p.cov && !restoring)
                for (uint32_t bb = b + 1; bb < b1; ++bb) atomicAdd(&p.cov[bb], 1u);
              ws.blocks -= b1 - b;                         // tiles b..b1-1 are not complete
              ws.reason = kReasonYield;
              ws.partial = b1 - b;                         // the epoch cannot complete (R23)
              leave = true;
              break;
            }
          }
        }
        mbar_wait(&s->qempty[qi], qph ^ 1u);
        s->tile_q[qi] = STOP;
        mbar_arrive(&s->qfull[qi]);
      }
    } else if (warp == 1) {
      if (lane == 0) {                                     // ---- MMA issuer
        uint32_t qi = 0, qph = 0, st = 0, ph = 0, acc = 0, aph = 0;
        uint32_t rph[2] = {0u, 0u};
        const uint32_t tmem0 = s->tmem_base;
        while (true) {
          mbar_wait(&s->qfull[qi], qph);
          const uint32_t b = s->tile_q[qi];
          const uint32_t kb0 = s->tile_kb0[qi];
          mbar_arrive(&s->qempty[qi]);
          if (++qi == QDEPTH) { qi = 0; qph ^= 1u; }
          if (b == STOP) break;
          mbar_wait(&s->tempty[acc], aph ^ 1u);            // epilogue drained this half
          if (kb0 > 0) { mbar_wait(&s->trest[acc], rph[acc]); rph[acc] ^= 1u; }   // restored
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          const uint32_t tmem = tmem0 + acc * BN;
          uint32_t kb = kb0;
          for (; kb < nk; ++kb) {
            mbar_wait(&s->full[st], ph);
            if (s->stage_stop[st]) {                       // stop marker: release it, commit
              mbar_arrive(&s->empty[st]);
              if (++st == STAGES) { st = 0; ph ^= 1u; }
              break;
            }
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            const uint32_t sa = smem_u32(base + st * kStage), sb = sa + kBytesA;
#pragma unroll
            for (uint32_t k = 0; k < BK / UMMA_K; ++k) {
              const uint64_t da = sdesc(sa + k * UMMA_K * 2), db = sdesc(sb + k * UMMA_K * 2);
              const uint32_t accum = (kb | k) ? 1u : 0u;   // kb0 > 0: continue the restored sum
              asm volatile(
                  "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
                  " tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n"
                  :: "r"(tmem), "l"(da), "l"(db), "r"(kIdesc), "r"(accum) : "memory");
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                         :: "r"(smem_u32(&s->empty[st])) : "memory");
            if (++st == STAGES) { st = 0; ph ^= 1u; }
          }
          s->acc_kend[acc] = kb;
          asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                       :: "r"(smem_u32(&s->tfull[acc])) : "memory");
          mbar_arrive(&s->tfull[acc]);                     // publishes acc_kend (release)
          if (++acc == 2) { acc = 0; aph ^= 1u; }
        }
      }
    } else if (warp >= 4) {                                // ---- epilogue (128 threads)
      const uint32_t q = warp - 4;
      const uint32_t rl = q * 32u + lane;                  // tile row (TMEM lane) of this thread
      uint32_t qi = 0, qph = 0, acc = 0, aph = 0, it = 0;
      while (true) {
        mbar_wait(&s->qfull[qi], qph);
        const uint32_t b = s->tile_q[qi];
        const uint32_t kb0 = s->tile_kb0[qi];
        __syncwarp();
        if (lane == 0) mbar_arrive(&s->qempty[qi]);
        if (++qi == QDEPTH) { qi = 0; qph ^= 1u; }
        if (b == STOP) break;
        int32_t tm, tn;
        tile_coords(b, gx, p_gy(g), tm, tn);
        const uint32_t tmem = s->tmem_base + acc * BN + ((q * 32u) << 16);
        if (kb0 > 0) {                                     // restore the spilled accumulator
          const float4* src = spill_slot(p);               // layout [col/4][row]: coalesced
#pragma unroll 1
          for (uint32_t c0 = 0; c0 < BN; c0 += 32) {
            uint32_t r[32];
#pragma unroll
            for (int j = 0; j < 8; ++j) {
              const float4 v = __ldcs(src + (size_t)(c0 / 4 + j) * BM + rl);
              r[4 * j] = __float_as_uint(v.x); r[4 * j + 1] = __float_as_uint(v.y);
              r[4 * j + 2] = __float_as_uint(v.z); r[4 * j + 3] = __float_as_uint(v.w);
            }
            tmem_st32(tmem + c0, r);
          }
          asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
          asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
          mbar_arrive(&s->trest[acc]);
        }
        mbar_wait(&s->tfull[acc], aph);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        if (s->acc_kend[acc] < nk) {                       // stopped inside the tile: spill
          float4* dst = spill_slot(p);
#pragma unroll 1
          for (uint32_t c0 = 0; c0 < BN; c0 += 32) {
            uint32_t r[32];
            tmem_ld32(tmem + c0, r);
#pragma unroll
            for (int j = 0; j < 8; ++j)
              __stcs(dst + (size_t)(c0 / 4 + j) * BM + rl,
                     make_float4(__uint_as_float(r[4 * j]), __uint_as_float(r[4 * j + 1]),
                                 __uint_as_float(r[4 * j + 2]), __uint_as_float(r[4 * j + 3])));
          }
        } else {
          store_bulk(&g.tma_c, epi_buf(q), tmem, 0, BN, tn * (int32_t)BN, tm * (int32_t)BM + (int32_t)(q * 32u), lane, it);
        }
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        mbar_arrive(&s->tempty[acc]);
        if (++acc == 2) { acc = 0; aph ^= 1u; }
      }
      bulk_wait_all(lane);
    }
    __syncthreads();
  }
};

// host side (gemm_tcgen05.cu)
cudaError_t gemm_worker_launch(const void* user_args, const WorkerParams& p, uint32_t W, cudaStream_t s, bool cov);
cudaError_t gemm_unwrapped_launch(const void* user_args, dim3 grid, uint32_t offset, uint32_t count, cudaStream_t s);
cudaError_t gemm_occupancy(int* k, bool cov);
const char* gemm_validate(const void* user_args, dim3 grid);

}  // namespace flep
