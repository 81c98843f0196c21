// gemm2_tcgen05.cuh — the dense-contraction body on CTA pairs (FLEP_BODY_GEMM_BF16_2SM):
// C = A·Bᵀ (A [M,K], B [N,K] bf16 row-major, K-major "TN"), fp32 accumulation in TMEM, bf16 out.
// Same operation as gemm_tcgen05.cuh (MM, Table 1), B200-native shape:
//
//   one original block = one 256x256 output tile, computed by a cluster of 2 CTAs on one TPC
//   with tcgen05.mma.cta_group::2 (M = 256, N = 256, K = 16): CTA r holds rows 128r..128r+127
//   of the A tile and of the B tile in its shared memory and receives rows 128r..128r+127 of the
//   256x256 accumulator in its TMEM. Per k-step (BK = 64) each CTA loads 16 KB of A and 16 KB of
//   B (the 1-CTA 128x256 tile loads 48 KB for the same MMA work per SM), so L2 -> SM operand
//   traffic per flop drops by a third and the tensor pipe is fed from both SMs' shared memory.
//
// Roles (8 warps per CTA):
//   leader warp 0 lane 0 : FLEP scheduling step (poll, fetch, exit accounting: the PAIR is the
//                          worker) + tile queue of both CTAs (its own by st.shared, the peer's by
//                          st.shared::cluster + a remote mbarrier arrive) + its TMA loads
//   peer warp 0 lane 0   : its TMA loads, tiles taken from its queue
//     both TMA loads of a stage complete on the LEADER's full barrier (cta_group::2 TMA)
//   leader warp 1 lane 0 : MMA issuer; commits free each stage / publish each accumulator to
//                          both CTAs (multicast commit)
//   warp 2               : TMEM allocator (cta_group::2) in both CTAs
//   warps 4..7           : epilogue of the CTA's 128 rows: tcgen05.ld -> bf16 -> global; then
//                          a (remote, for the peer) arrive on the leader's accumulator-empty
//                          barrier
// Preemption granularity: one tile (the pair polls between chunks), or — registered with
// FLEP_KFLAG_IN_TILE — a few k-steps: the pair stops inside a tile and spills both 128-row halves
// of its accumulator (worker_pipeline below, R21 + R32). A spatial request releases a pair iff it
// names either of its SMs (a pair cannot split), R32.
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <cstdint>

#include "../../include/flep.h"
#include "flep_device.cuh"
#include "gemm_tcgen05.cuh"

namespace flep {

struct Gemm2Args {
  CUtensorMap tma_a;           // A [M,K] bf16, box {64, 128}, SWIZZLE_128B
  CUtensorMap tma_b;           // B [N,K] bf16, box {64, 128}, SWIZZLE_128B
  CUtensorMap tma_c;           // C [M,N] bf16, box {64, 32}, SWIZZLE_128B (epilogue bulk stores)
  __nv_bfloat16* c;            // C [M,N] bf16 row-major
  uint32_t m, n, k;
};

template <uint32_t kBN>
struct Gemm2T {
  static constexpr int kThreads = 256;
  // BN = 256: the 256x256 pair tile, two TMEM accumulators (the epilogue of one tile overlaps the
  // next tile's MMAs), 6 stages of 32 KB. BN = 512 (the wide tile, FLEP_BODY_GEMM_BF16_2SM_W): a
  // 256x512 pair tile as two N = 256 MMAs per k-slice into one 512-column accumulator, 4 stages of
  // 48 KB: per k-step each SM loads 16 KB of A and 32 KB of B for twice the MMA work, so L2 -> SM
  // operand traffic per flop drops by a quarter more (the tensor pipe is ~96 % active in both
  // shapes at 8192^3; the wide tile's lower fabric traffic is what keeps the clock up under the
  // power cap).
  static constexpr uint32_t BM = 128, BN = kBN, BK = 64, UMMA_K = 16, MMA_N = 256;
  static constexpr uint32_t NH = BN / MMA_N;                   // MMAs per k-slice (B halves of 128 rows per CTA)
  static constexpr uint32_t NACC = 512 / BN;                   // TMEM accumulators (512 columns in all)
  static constexpr uint32_t STAGES = NH == 1 ? 6 : 4;
  static_assert(NH == 1 || NH == 2, "BN is 256 or 512");
  static constexpr uint32_t TM = 2 * BM;                       // tile rows of the pair
  static constexpr uint32_t kHalfB = 128 * BK * 2;             // one 128-row B box (16 KB)
  static constexpr uint32_t kBytesA = BM * BK * 2, kBytesB = NH * kHalfB, kStage = kBytesA + kBytesB;
  static constexpr uint32_t kTmemCols = 512;                   // NACC accumulators of 128 lanes x BN columns
  static constexpr size_t kSpill = kSpillBytes * NH;           // one CTA's fp32 128 x BN half
  static constexpr uint32_t QDEPTH = 4;
  static constexpr uint32_t kQConsumers = 10;                  // leader: MMA + 4 epilogue warps; peer: producer + 4
  // epilogue staging: per epilogue warp two 4 KB buffers of 32 rows x 64 bf16 columns (128-B
  // rows, SWIZZLE_128B) that a bulk tensor store writes to C
  static constexpr uint32_t kEpiBuf = 32 * 128;
  static constexpr size_t kDynSmem = 1024 + STAGES * kStage + 1024 + 4 * 2 * kEpiBuf;
  static_assert(kDynSmem <= 232448, "shared memory per block");
  static constexpr uint32_t STOP = 0xffffffffu;
  static constexpr uint32_t STOP_PARTIAL = 0xfffffffeu;         // in-tile: the last tile was stopped

  struct State {
    uint64_t full[STAGES], empty[STAGES];
    uint64_t tfull[2], tempty[2];
    uint64_t qfull[QDEPTH], qempty[QDEPTH];
    uint64_t trest[2];                // in-tile: both CTAs restored a spilled half (leader's, count 8)
    uint32_t tile_q[QDEPTH];
    uint32_t tile_kb0[QDEPTH];        // in-tile: first k-step of the tile (> 0: continue a spill)
    uint32_t stage_stop[STAGES];      // in-tile: this stage is a stop marker (leader)
    uint32_t lic;                     // in-tile (peer): k-step loads the leader has licensed
    uint32_t stop_at;                 // in-tile (peer): the licence count at which loads stop
    uint32_t tmem_base;
    uint32_t smid;
  };

  __device__ static uint8_t* ring() {
    extern __shared__ uint8_t dsmem[];
    const uint32_t a = static_cast<uint32_t>(__cvta_generic_to_shared(dsmem));
    return dsmem + (((a + 1023u) & ~1023u) - a);
  }
  __device__ static State* state() { return reinterpret_cast<State*>(ring() + STAGES * kStage); }
  __device__ static uint8_t* epi_buf(uint32_t q, uint32_t bi) {
    return ring() + STAGES * kStage + 1024 + (2 * q + bi) * kEpiBuf;
  }
  __device__ static uint32_t su32(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }
  __device__ static uint32_t rank() { uint32_t r; asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r)); return r; }
  // shared::cluster address of `local` in CTA `r` of the cluster
  __device__ static uint32_t peer_addr(const void* local, uint32_t r) {
    uint32_t a; asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(a) : "r"(su32(local)), "r"(r)); return a;
  }
  __device__ static void cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n barrier.cluster.wait.acquire.aligned;" ::: "memory");
  }
  __device__ static void mbar_init(uint64_t* b, uint32_t n) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(su32(b)), "r"(n) : "memory");
  }
  // waits that may follow remote (cluster-scope) arrivals acquire at cluster scope
  __device__ static void wait(uint64_t* b, uint32_t parity) {
    asm volatile(
        "{\n .reg .pred p;\n W: mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%0], %1;\n"
        " @!p bra W;\n}\n" :: "r"(su32(b)), "r"(parity) : "memory");
  }
  __device__ static bool test_wait(uint64_t* b, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.test_wait.parity.acquire.cluster.shared::cta.b64 p, [%1], %2;\n"
        " selp.u32 %0, 1, 0, p;\n}\n" : "=r"(ok) : "r"(su32(b)), "r"(parity) : "memory");
    return ok != 0;
  }
  __device__ static void arrive_local(uint64_t* b) {
    asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" :: "r"(su32(b)) : "memory");
  }
  __device__ static void arrive_remote(uint32_t cluster_addr) {
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" :: "r"(cluster_addr) : "memory");
  }
  __device__ static void expect_tx(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su32(b)), "r"(bytes) : "memory");
  }
  // cta_group::2 TMA: the data lands in this CTA's smem, completion is counted on the leader's
  // barrier (cluster address)
  __device__ static void tma_2sm(const CUtensorMap* map, void* dst, uint32_t bar_cluster, int32_t x, int32_t y) {
    asm volatile(
        "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
        :: "r"(su32(dst)), "l"(reinterpret_cast<uint64_t>(map)), "r"(bar_cluster), "r"(x), "r"(y) : "memory");
  }
  __device__ static uint64_t sdesc(uint32_t saddr) {   // as GemmBody::sdesc (K-major, SWIZZLE_128B)
    return (uint64_t)((saddr >> 4) & 0x3FFFu) | ((uint64_t)1u << 16) | ((uint64_t)(1024u >> 4) << 32) |
           ((uint64_t)1u << 46) | ((uint64_t)2u << 61);
  }
  // kind::f16, D f32, A/B bf16 K-major, N = 256, M = 256 (the pair)
  static constexpr uint32_t kIdesc = (1u << 4) | (1u << 7) | (1u << 10) | ((MMA_N >> 3) << 17) | ((TM >> 4) << 24);
  // this CTA's B rows of a k-step: for MMA h, rows tn*BN + 256h + 128r .. +127 (a cta_group::2
  // MMA with N = 256 takes B rows 0..127 from the leader's and 128..255 from the peer's smem)
  __device__ static void load_b(const Gemm2Args& g, uint8_t* sb, uint32_t fb, uint32_t kb, int32_t tn, uint32_t r) {
#pragma unroll
    for (uint32_t h = 0; h < NH; ++h)
      tma_2sm(&g.tma_b, sb + h * kHalfB, fb, (int32_t)(kb * BK), tn * (int32_t)BN + (int32_t)(h * MMA_N + r * 128));
  }
  // the MMAs of one k-step for column half h of the wide tile (B box h)
  __device__ static void mma_half(uint32_t tmem_h, uint32_t sa, uint32_t kb, uint32_t h) {
    const uint32_t sb = sa + kBytesA + h * kHalfB;
#pragma unroll
    for (uint32_t k = 0; k < BK / UMMA_K; ++k) {
      const uint64_t da = sdesc(sa + k * UMMA_K * 2), db = sdesc(sb + k * UMMA_K * 2);
      const uint32_t accum = (kb | k) ? 1u : 0u;
      asm volatile(
          "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
          " tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n}\n"
          :: "r"(tmem_h), "l"(da), "l"(db), "r"(kIdesc), "r"(accum) : "memory");
    }
  }
  __device__ static void commit_multicast(uint64_t* b) {   // arrives on b in both CTAs of the pair
    asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                 :: "r"(su32(b)), "h"((uint16_t)3) : "memory");
  }
  // the MMAs of one k-step (stage at sa: A, then the NH B boxes)
  __device__ static void mma_kstep(uint32_t tmem, uint32_t sa, uint32_t kb) {
    const uint32_t sb = sa + kBytesA;
#pragma unroll
    for (uint32_t k = 0; k < BK / UMMA_K; ++k) {
      const uint64_t da = sdesc(sa + k * UMMA_K * 2);
      const uint32_t accum = (kb | k) ? 1u : 0u;
#pragma unroll
      for (uint32_t h = 0; h < NH; ++h) {
        const uint64_t db = sdesc(sb + h * kHalfB + k * UMMA_K * 2);
        asm volatile(
            "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
            " tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n}\n"
            :: "r"(tmem + h * MMA_N), "l"(da), "l"(db), "r"(kIdesc), "r"(accum) : "memory");
      }
    }
  }

  // original block b -> 256x256 tile (tm, tn): bands of GROUP tile-rows, column-major inside
  static constexpr uint32_t GROUP = 8;
  __device__ static void tile_coords(uint32_t b, uint32_t gx, uint32_t gy, int32_t& tm, int32_t& tn) {
    const uint32_t band = GROUP * gx;
    const uint32_t grp = b / band, r = b % band;
    const uint32_t rows = min(GROUP, gy - grp * GROUP);
    tm = (int32_t)(grp * GROUP + r % rows);
    tn = (int32_t)(r / rows);
  }

  // setup: barriers, TMEM (both CTAs), cluster barrier so that no remote access precedes init
  __device__ static void setup() {
    State* s = state();
    const uint32_t warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) {
      for (uint32_t i = 0; i < STAGES; ++i) { mbar_init(&s->full[i], 1); mbar_init(&s->empty[i], 1); }
      for (uint32_t i = 0; i < 2; ++i) { mbar_init(&s->tfull[i], 1); mbar_init(&s->tempty[i], 8); }
      for (uint32_t i = 0; i < QDEPTH; ++i) { mbar_init(&s->qfull[i], 1); mbar_init(&s->qempty[i], kQConsumers); }
      // in-tile: trest counts one arrive per epilogue warp of both CTAs
      for (uint32_t i = 0; i < 2; ++i) mbar_init(&s->trest[i], 8);
      for (uint32_t i = 0; i < STAGES; ++i) s->stage_stop[i] = 0;
      s->lic = 0; s->stop_at = 0xffffffffu;
      s->smid = smid_reg();
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 2) {
      asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;"
                   :: "r"(su32(&s->tmem_base)), "r"(kTmemCols) : "memory");
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    cluster_sync();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  }
  __device__ static void teardown() {
    State* s = state();
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    cluster_sync();                 // no CTA of the pair touches the other's smem / TMEM any more
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if ((threadIdx.x >> 5) == 2)
      asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" :: "r"(s->tmem_base), "r"(kTmemCols) : "memory");
  }

  // Epilogue of one warp's 32 accumulator rows, columns [c_begin, c_end): GemmBody::store_bulk
  // (TMEM -> bf16 -> the warp's two SWIZZLE_128B staging buffers -> bulk tensor stores of C)
  __device__ static void store_cols(const Gemm2Args& g, uint32_t tmem_w, uint32_t c_begin, uint32_t c_end,
                                    int32_t x0, int32_t y0, uint32_t q, uint32_t lane, uint32_t& it) {
    static_assert(kEpiBuf == GemmBody::kEpiBuf, "staging buffer size");
    GemmBody::store_bulk(&g.tma_c, epi_buf(q, 0), tmem_w, c_begin, c_end, x0, y0, lane, it);
  }
  __device__ static void bulk_wait_all(uint32_t lane) { GemmBody::bulk_wait_all(lane); }

  // The pair's pipeline. Next(b0, b1) is called by the leader's scheduling thread: it returns
  // false when the pair must stop, else the next chunk [b0, b1) of tiles. Returns after both
  // CTAs drained every tile handed out.
  template <class Next>
  __device__ static void pipeline(const Gemm2Args& g, uint32_t gx, uint32_t gy, Next next) {
    State* s = state();
    uint8_t* base = ring();
    const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31u;
    const uint32_t r = rank();
    const bool leader = r == 0;
    const uint32_t nk = g.k / BK;
    if (warp == 0 && lane == 0) {                       // ---- scheduler (leader) + TMA producer
      uint32_t qi = 0, qph = 0, st = 0, ph = 0;
      const uint32_t full0 = peer_addr(&s->full[0], 0);  // the leader's full barriers
      auto load_tile = [&](uint32_t tile) {
        int32_t tm, tn;
        tile_coords(tile, gx, gy, tm, tn);
        for (uint32_t kb = 0; kb < nk; ++kb) {
          wait(&s->empty[st], ph ^ 1u);
          uint8_t* sa = base + st * kStage;
          if (leader) expect_tx(&s->full[st], 2 * kStage);
          const uint32_t fb = full0 + st * 8u;
          tma_2sm(&g.tma_a, sa, fb, (int32_t)(kb * BK), tm * (int32_t)TM + (int32_t)(r * BM));
          load_b(g, sa + kBytesA, fb, kb, tn, r);
          if (++st == STAGES) { st = 0; ph ^= 1u; }
        }
      };
      if (leader) {
        auto push = [&](uint32_t tile) {                 // into the queues of both CTAs
          wait(&s->qempty[qi], qph ^ 1u);
          s->tile_q[qi] = tile;
          asm volatile("st.shared::cluster.u32 [%0], %1;" :: "r"(peer_addr(&s->tile_q[qi], 1)), "r"(tile) : "memory");
          arrive_local(&s->qfull[qi]);
          arrive_remote(peer_addr(&s->qfull[qi], 1));
          if (++qi == QDEPTH) { qi = 0; qph ^= 1u; }
        };
        uint32_t b0, b1;
        while (next(b0, b1)) {
          for (uint32_t b = b0; b < b1; ++b) { push(b); load_tile(b); }
        }
        push(STOP);
      } else {
        while (true) {
          wait(&s->qfull[qi], qph);
          const uint32_t tile = s->tile_q[qi];
          arrive_remote(peer_addr(&s->qempty[qi], 0));
          if (++qi == QDEPTH) { qi = 0; qph ^= 1u; }
          if (tile == STOP) break;
          load_tile(tile);
        }
      }
    } else if (warp == 1 && lane == 0 && leader) {      // ---- MMA issuer (leader only)
      uint32_t qi = 0, qph = 0, st = 0, ph = 0, acc = 0, aph = 0;
      const uint32_t tmem0 = s->tmem_base;
      while (true) {
        wait(&s->qfull[qi], qph);
        const uint32_t tile = s->tile_q[qi];
        arrive_local(&s->qempty[qi]);
        if (++qi == QDEPTH) { qi = 0; qph ^= 1u; }
        if (tile == STOP) break;
        if constexpr (NH == 1) {
          wait(&s->tempty[acc], aph ^ 1u);               // both CTAs' epilogues drained this accumulator
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          const uint32_t tmem = tmem0 + acc * BN;
          for (uint32_t kb = 0; kb < nk; ++kb) {
            wait(&s->full[st], ph);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            mma_kstep(tmem, su32(base + st * kStage), kb);
            commit_multicast(&s->empty[st]);             // frees stage st in both CTAs
            if (++st == STAGES) { st = 0; ph ^= 1u; }
          }
        } else {
          // Wide tile, one accumulator: tempty[h] says column half h is drained. The MMAs of
          // half 0 start as soon as half 0 is drained and run up to STAGES k-steps ahead of
          // half 1's while the epilogue still drains half 1 (a stage is freed once both halves
          // consumed it); each half still accumulates its k-steps in order (bit-identical).
          wait(&s->tempty[0], aph ^ 1u);
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          uint32_t kb0 = 0, kb1 = 0, st0 = st, ph0 = ph;
          bool h1 = false;
          while (kb1 < nk) {
            if (!h1 && test_wait(&s->tempty[1], aph ^ 1u)) {
              h1 = true;
              asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            }
            if (h1 && kb1 < kb0) {
              mma_half(tmem0 + MMA_N, su32(base + st * kStage), kb1, 1);
              commit_multicast(&s->empty[st]);
              if (++st == STAGES) { st = 0; ph ^= 1u; }
              ++kb1;
            } else if (kb0 < nk && kb0 - kb1 < STAGES) {
              wait(&s->full[st0], ph0);
              asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
              mma_half(tmem0, su32(base + st0 * kStage), kb0, 0);
              if (++st0 == STAGES) { st0 = 0; ph0 ^= 1u; }
              ++kb0;
            } else {
              wait(&s->tempty[1], aph ^ 1u);
              h1 = true;
              asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            }
          }
        }
        // the accumulator is complete in both CTAs' TMEM
        commit_multicast(&s->tfull[NH == 1 ? acc : 0u]);
        if (++acc == NACC) { acc = 0; aph ^= 1u; }
      }
    } else if (warp >= 4) {                              // ---- epilogue: this CTA's 128 rows
      const uint32_t q = warp - 4;
      uint32_t qi = 0, qph = 0, acc = 0, aph = 0, it = 0;
      const uint32_t tempty0 = peer_addr(&s->tempty[0], 0);
      while (true) {
        wait(&s->qfull[qi], qph);
        const uint32_t tile = s->tile_q[qi];
        __syncwarp();
        if (lane == 0) {
          if (leader) arrive_local(&s->qempty[qi]);
          else arrive_remote(peer_addr(&s->qempty[qi], 0));
        }
        if (++qi == QDEPTH) { qi = 0; qph ^= 1u; }
        if (tile == STOP) break;
        int32_t tm, tn;
        tile_coords(tile, gx, gy, tm, tn);
        wait(&s->tfull[acc], aph);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint32_t tmem = s->tmem_base + acc * BN + ((q * 32u) << 16);
        const int32_t x0 = tn * (int32_t)BN, y0 = tm * (int32_t)TM + (int32_t)(r * BM + q * 32u);
        // NH == 1: one arrive on tempty[acc] after the whole tile; NH == 2: one per column half
#pragma unroll 1
        for (uint32_t h = 0; h < NH; ++h) {
          store_cols(g, tmem, h * MMA_N, (h + 1) * MMA_N, x0, y0, q, lane, it);
          asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
          __syncwarp();
          const uint32_t e = NH == 1 ? acc : h;
          if (lane == 0) {
            if (leader) arrive_local(&s->tempty[e]);
            else arrive_remote(tempty0 + e * 8u);
          }
        }
        if (++acc == NACC) { acc = 0; aph ^= 1u; }
      }
      bulk_wait_all(lane);
    }
  }

  // ---- the FLEP worker's pipeline with in-tile preemption (R32 + R21) --------------------------
  // As `pipeline`, plus: the leader's producer polls the control word every kInTilePoll k-steps
  // inside a tile; the peer's producer issues a k-step's loads only once the leader has licensed
  // it (a running licence count, kLicSlack ahead of the leader's own loads, written into the
  // peer's shared memory), so at a stop both CTAs load exactly the same k-steps: the leader tells
  // the peer the last licensed count, loads up to it itself, sends a stop
  // marker through its stage ring, the MMA commits the partial accumulator and publishes the
  // k-steps it holds to both CTAs, both epilogues spill their 128-row halves to the pair's slots,
  // and the leader records {tile, next k-step, chunk end}. The pair with the same index in the
  // next epoch restores both halves (tcgen05.st) and continues the k-loop: every k-step of every
  // tile is accumulated once, in order (bit-identical to an uninterrupted run).
  static constexpr uint32_t kInTilePoll = 4, kMinLeft = 4;
  // the peer may run kLicSlack loads ahead of the leader; a stop then lets the leader catch up to
  // the licensed count (kLicSlack more k-steps, < kMinLeft so they are in the same tile)
#ifndef FLEP_GEMM2_LIC_SLACK
#define FLEP_GEMM2_LIC_SLACK 2
#endif
  static constexpr uint32_t kLicSlack = FLEP_GEMM2_LIC_SLACK;
  static_assert(kLicSlack <= kMinLeft, "the catch-up loads must stay inside the tile");
  __device__ static float4* spill_slot(const WorkerParams& p, uint32_t wid, uint32_t r) {
    return reinterpret_cast<float4*>(reinterpret_cast<uint8_t*>(p.partial) + partial_header_bytes(2 * p.workers) +
                                     (size_t)(2 * wid + r) * kSpill);
  }
  template <bool kCov, class Fetch>
  __device__ static void worker_pipeline(const Gemm2Args& g, const WorkerParams& p, WorkerShared& ws,
                                         uint32_t wid, uint32_t yield_sm, Fetch fetch) {
    State* s = state();
    uint8_t* base = ring();
    const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31u;
    const uint32_t r = rank();
    const bool leader = r == 0;
    const uint32_t nk = g.k / BK;
    const bool in_tile = p.partial != nullptr;
    const uint32_t gx = p.gx, gy = p.gy;
    if (warp == 0 && lane == 0) {                       // ---- scheduler (leader) + TMA producers
      uint32_t qi = 0, qph = 0, st = 0, ph = 0, q = 0;  // q: k-step loads issued (licence count)
      const uint32_t full0 = peer_addr(&s->full[0], 0);
      if (leader) {
        const uint32_t lic_peer = peer_addr(&s->lic, 1), stop_peer = peer_addr(&s->stop_at, 1);
        auto push = [&](uint32_t tile, uint32_t kb0) {
          wait(&s->qempty[qi], qph ^ 1u);
          s->tile_q[qi] = tile;
          s->tile_kb0[qi] = kb0;
          asm volatile("st.shared::cluster.u32 [%0], %1;" :: "r"(peer_addr(&s->tile_q[qi], 1)), "r"(tile) : "memory");
          asm volatile("st.shared::cluster.u32 [%0], %1;" :: "r"(peer_addr(&s->tile_kb0[qi], 1)), "r"(kb0) : "memory");
          arrive_local(&s->qfull[qi]);
          arrive_remote(peer_addr(&s->qfull[qi], 1));
          if (++qi == QDEPTH) { qi = 0; qph ^= 1u; }
        };
        PartialTile* mine = in_tile ? reinterpret_cast<PartialTile*>(p.partial) + wid : nullptr;
        uint32_t rb0 = STOP, rb1 = 0, rkb = 0, q_stop = 0;
        bool leave = false, stopping = false, stopped_in_tile = false;
        SchedState sch;
        if (in_tile) asm volatile("st.relaxed.cluster.shared::cluster.u32 [%0], %1;" :: "r"(lic_peer), "r"(kLicSlack) : "memory");
        if (in_tile) {
          if (p.epoch == p.gen_first) {
            mine->valid = 0;
          } else {
            const PartialTile e = *mine;
            if (e.valid) {
              sch.first = false;
              if (should_yield(poll_ctrl(p), p, yield_sm)) {      // entry check (a2)
                ws.reason = kReasonYield;
                ws.partial = e.b_end - e.b;
                leave = true;
              } else {
                rb0 = e.b; rb1 = e.b_end; rkb = e.kb;
                mine->valid = 0;
                ws.blocks += e.b_end - e.b;
              }
            }
          }
        }
        while (!leave) {
          uint32_t b0, b1, kbs = 0;
          bool restoring = false;
          if (rb0 != STOP) {
            b0 = rb0; b1 = rb1; kbs = rkb; restoring = true; rb0 = STOP;
          } else {
            if (!fetch(sch, b0, b1)) break;
          }
          for (uint32_t b = b0; b < b1; ++b) {
            const uint32_t kb0 = (restoring && b == b0) ? kbs : 0u;
            push(b, kb0);
            if (kCov && !restoring) atomicAdd(&p.cov[b], 1u);
            int32_t tm, tn;
            tile_coords(b, gx, gy, tm, tn);
            uint32_t kb = kb0, pend = 0;
            bool pend_valid = false, stop = false;
            for (; kb < nk; ++kb) {
              if (in_tile) {
                if (stopping) {                        // catching up to the licensed count
                  if (q == q_stop) { stop = true; break; }
                } else {                               // amortised in-tile poll (as GemmBody)
                  const uint32_t j = kb - kb0;
                  if (pend_valid && j % kInTilePoll == kInTilePoll / 2) {
                    pend_valid = false;
                    if (nk - kb > kMinLeft && should_yield(pend, p, yield_sm)) {
                      // the peer loads nothing from licence q_stop on
                      stopping = true;
                      q_stop = q + kLicSlack;
                      asm volatile("st.relaxed.cluster.shared::cluster.u32 [%0], %1;" :: "r"(stop_peer), "r"(q_stop) : "memory");
                      if (q == q_stop) { stop = true; break; }
                    }
                  }
                  if (j % kInTilePoll == 0 && j > 0) { pend = poll_ctrl(p); pend_valid = true; }
                }
              }
              wait(&s->empty[st], ph ^ 1u);
              s->stage_stop[st] = 0u;
              uint8_t* sa = base + st * kStage;
              expect_tx(&s->full[st], 2 * kStage);
              const uint32_t fb = full0 + st * 8u;
              tma_2sm(&g.tma_a, sa, fb, (int32_t)(kb * BK), tm * (int32_t)TM);
              load_b(g, sa + kBytesA, fb, kb, tn, 0);
              ++q;
              // the licence orders nothing else (relaxed: a release here fences every k-step)
              if (in_tile && !stopping)
                asm volatile("st.relaxed.cluster.shared::cluster.u32 [%0], %1;" :: "r"(lic_peer), "r"(q + kLicSlack) : "memory");
              if (++st == STAGES) { st = 0; ph ^= 1u; }
            }
            if (stop) {
              // both CTAs loaded k-steps < kb; a data-less stop marker ends the MMA's tile
              wait(&s->empty[st], ph ^ 1u);
              s->stage_stop[st] = 1u;
              arrive_local(&s->full[st]);
              if (++st == STAGES) { st = 0; ph ^= 1u; }
              mine->b = b; mine->kb = kb; mine->b_end = b1; mine->valid = 1;
              if (kCov && !restoring)
                for (uint32_t bb = b + 1; bb < b1; ++bb) atomicAdd(&p.cov[bb], 1u);
              ws.blocks -= b1 - b;
              ws.reason = kReasonYield;
              ws.partial = b1 - b;
              leave = stopped_in_tile = true;
              break;
            }
          }
        }
        push(stopped_in_tile ? STOP_PARTIAL : STOP, 0);
      } else {                                         // peer producer
        while (true) {
          wait(&s->qfull[qi], qph);
          const uint32_t tile = s->tile_q[qi];
          const uint32_t kb0 = s->tile_kb0[qi];
          arrive_remote(peer_addr(&s->qempty[qi], 0));
          if (++qi == QDEPTH) { qi = 0; qph ^= 1u; }
          if (tile >= STOP_PARTIAL) break;
          int32_t tm, tn;
          tile_coords(tile, gx, gy, tm, tn);
          bool stopped = false;
          for (uint32_t kb = kb0; kb < nk; ++kb) {
            if (in_tile) {                             // wait for the licence of load q (or a stop)
              while (true) {
                uint32_t l, sa_;
                asm volatile("ld.relaxed.cluster.shared::cta.u32 %0, [%1];" : "=r"(l) : "r"(su32(&s->lic)) : "memory");
                if (l > q) break;
                asm volatile("ld.relaxed.cluster.shared::cta.u32 %0, [%1];" : "=r"(sa_) : "r"(su32(&s->stop_at)) : "memory");
                if (sa_ == q) { stopped = true; break; }
              }
              if (stopped) break;
            }
            wait(&s->empty[st], ph ^ 1u);
            uint8_t* sa = base + st * kStage;
            const uint32_t fb = full0 + st * 8u;
            tma_2sm(&g.tma_a, sa, fb, (int32_t)(kb * BK), tm * (int32_t)TM + (int32_t)BM);
            load_b(g, sa + kBytesA, fb, kb, tn, 1);
            ++q;
            if (++st == STAGES) { st = 0; ph ^= 1u; }
          }
          // after a stop the leader pushes STOP next: the loop ends there (the leader's ring is one
          // stage ahead, the stop marker; the pair leaves, so the rings are not used again)
        }
      }
    } else if (warp == 1 && lane == 0 && leader) {      // ---- MMA issuer (leader only)
      uint32_t qi = 0, qph = 0, st = 0, ph = 0, acc = 0, aph = 0;
      uint32_t rph[2] = {0u, 0u};
      const uint32_t tmem0 = s->tmem_base;
      while (true) {
        wait(&s->qfull[qi], qph);
        const uint32_t tile = s->tile_q[qi];
        const uint32_t kb0 = s->tile_kb0[qi];
        arrive_local(&s->qempty[qi]);
        if (++qi == QDEPTH) { qi = 0; qph ^= 1u; }
        if (tile >= STOP_PARTIAL) break;
        wait(&s->tempty[acc], aph ^ 1u);
        if constexpr (NH == 2) wait(&s->tempty[1], aph ^ 1u);   // wide tile: both column halves drained
        if (kb0 > 0) { wait(&s->trest[acc], rph[acc]); rph[acc] ^= 1u; }   // both halves restored
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint32_t tmem = tmem0 + acc * BN;
        uint32_t kb = kb0;
        for (; kb < nk; ++kb) {
          wait(&s->full[st], ph);
          if (s->stage_stop[st]) {                     // stop marker (the pair leaves: the rings
            arrive_local(&s->empty[st]);               // are not used again)
            if (++st == STAGES) { st = 0; ph ^= 1u; }
            break;
          }
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          mma_kstep(tmem, su32(base + st * kStage), kb);
          asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                       :: "r"(su32(&s->empty[st])), "h"((uint16_t)3) : "memory");
          if (++st == STAGES) { st = 0; ph ^= 1u; }
        }
        asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                     :: "r"(su32(&s->tfull[acc])), "h"((uint16_t)3) : "memory");
        if (++acc == NACC) { acc = 0; aph ^= 1u; }
      }
    } else if (warp >= 4) {                              // ---- epilogue: this CTA's 128 rows
      const uint32_t qw = warp - 4;
      const uint32_t rl = qw * 32u + lane;
      uint32_t qi = 0, qph = 0, acc = 0, aph = 0, it = 0;
      const uint32_t tempty0 = peer_addr(&s->tempty[0], 0), trest0 = peer_addr(&s->trest[0], 0);
      while (true) {
        wait(&s->qfull[qi], qph);
        const uint32_t tile = s->tile_q[qi];
        const uint32_t kb0 = s->tile_kb0[qi];
        __syncwarp();
        if (lane == 0) {
          if (leader) arrive_local(&s->qempty[qi]);
          else arrive_remote(peer_addr(&s->qempty[qi], 0));
        }
        if (++qi == QDEPTH) { qi = 0; qph ^= 1u; }
        if (tile >= STOP_PARTIAL) break;
        int32_t tm, tn;
        tile_coords(tile, gx, gy, tm, tn);
        const uint32_t tmem = s->tmem_base + acc * BN + ((qw * 32u) << 16);
        if (kb0 > 0) {                                   // restore this CTA's spilled half
          const float4* src = spill_slot(p, wid, r);     // layout [col/4][row]: coalesced
#pragma unroll 1
          for (uint32_t c0 = 0; c0 < BN; c0 += 32) {
            uint32_t v[32];
#pragma unroll
            for (int j = 0; j < 8; ++j) {
              const float4 f = __ldcs(src + (size_t)(c0 / 4 + j) * BM + rl);
              v[4 * j] = __float_as_uint(f.x); v[4 * j + 1] = __float_as_uint(f.y);
              v[4 * j + 2] = __float_as_uint(f.z); v[4 * j + 3] = __float_as_uint(f.w);
            }
            GemmBody::tmem_st32(tmem + c0, v);
          }
          asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
          asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
          __syncwarp();
          if (lane == 0) {
            if (leader) arrive_local(&s->trest[acc]);
            else arrive_remote(trest0 + acc * 8u);
          }
        }
        wait(&s->tfull[acc], aph);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        // stopped inside the tile iff the queue's next entry is STOP_PARTIAL (a stop is always
        // the pair's last tile; the leader pushes the next entry before this tile's MMAs end, so
        // the peek costs nothing; a remote publish from the MMA thread would fence its pipeline)
        wait(&s->qfull[qi], qph);
        if (s->tile_q[qi] == STOP_PARTIAL) {
          float4* dst = spill_slot(p, wid, r);
#pragma unroll 1
          for (uint32_t c0 = 0; c0 < BN; c0 += 32) {
            uint32_t v[32];
            GemmBody::tmem_ld32(tmem + c0, v);
#pragma unroll
            for (int j = 0; j < 8; ++j)
              __stcs(dst + (size_t)(c0 / 4 + j) * BM + rl,
                     make_float4(__uint_as_float(v[4 * j]), __uint_as_float(v[4 * j + 1]),
                                 __uint_as_float(v[4 * j + 2]), __uint_as_float(v[4 * j + 3])));
          }
        } else {
          store_cols(g, tmem, 0, BN, tn * (int32_t)BN, tm * (int32_t)TM + (int32_t)(r * BM + qw * 32u), qw, lane, it);
        }
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncwarp();
        if (lane == 0) {
          if (leader) arrive_local(&s->tempty[acc]);
          else arrive_remote(tempty0 + acc * 8u);
          if constexpr (NH == 2) {                       // wide tile: tempty[1] = column half 1
            if (leader) arrive_local(&s->tempty[1]);
            else arrive_remote(tempty0 + 8u);
          }
        }
        if (++acc == NACC) { acc = 0; aph ^= 1u; }
      }
      bulk_wait_all(lane);
    }
  }
};
using Gemm2 = Gemm2T<256>;
using Gemm2W = Gemm2T<512>;

// Worker (the PAIR is the FLEP worker: wid = cluster index, W = pairs). The leader runs the
// scheduling step of flep_worker (next_chunk: poll every K chunks, fetch C tiles, exit event);
// the spatial check uses the pair's lower-ranked SM so that a request naming either SM releases it.
template <class G, bool kCoverage>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(256, 1)
flep_gemm2_worker(const __grid_constant__ Gemm2Args g, const WorkerParams p) {
  __shared__ WorkerShared ws;
  const uint32_t wid = blockIdx.x >> 1;
  const bool leader = G::rank() == 0;
  if (threadIdx.x == 0) {
    ws.sm = smid_reg(); ws.t_entry = gtimer(); ws.blocks = 0; ws.reason = 0;
    ws.counted = 0; ws.last = 0; ws.ev_raw = 0; ws.ev_part = 0; ws.partial = 0;
    if (wid == 0 && leader && p.started_hint && p.status) st_relaxed_sys(&p.status->started, p.epoch);
  }
  G::setup();
  uint32_t yield_sm = 0;
  if (leader && threadIdx.x == 0) {                    // the pair's SM with the lower rank (spatial)
    uint32_t peer_sm;
    asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(peer_sm) : "r"(G::peer_addr(&G::state()->smid, 1)) : "memory");
    yield_sm = p.rank[peer_sm] < p.rank[ws.sm] ? peer_sm : ws.sm;
    ws.sm = yield_sm;                                  // the worker record names the deciding SM
  }
  if (p.partial) {                                     // in-tile preemption (R21 on the pair)
    G::template worker_pipeline<kCoverage>(g, p, ws, wid, yield_sm, [&](SchedState& st, uint32_t& b0, uint32_t& b1) {
      b0 = next_chunk(p, st, ws, wid, yield_sm);
      if (b0 == 0xffffffffu) return false;
      b1 = min(b0 + p.chunk, p.n_blocks);
      return true;
    });
  } else {
    SchedState st;
    G::pipeline(g, p.gx, p.gy, [&](uint32_t& b0, uint32_t& b1) {
      b0 = next_chunk(p, st, ws, wid, yield_sm);
      if (b0 == 0xffffffffu) return false;
      b1 = min(b0 + p.chunk, p.n_blocks);
      if (kCoverage)
        for (uint32_t b = b0; b < b1; ++b) atomicAdd(&p.cov[b], 1u);
      return true;
    });
  }
  G::teardown();
  if (leader && threadIdx.x == 0) worker_exit(p, ws, wid);
}

// The original kernel (unwrapped twin): one pair per tile.
template <class G>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(256, 1)
flep_gemm2_unwrapped(const __grid_constant__ Gemm2Args g, uint32_t gx, uint32_t gy, uint32_t offset) {
  G::setup();
  const uint32_t b = offset + (blockIdx.x >> 1) + (gridDim.x >> 1) * blockIdx.y;
  bool given = false;
  G::pipeline(g, gx, gy, [&](uint32_t& b0, uint32_t& b1) {
    if (given) return false;
    given = true; b0 = b; b1 = b + 1;
    return true;
  });
  G::teardown();
}

// Kernel slicing with the device check (R31): one pair per tile of the slice; every CTA follows
// the slice's one decision (taken by the first CTA of the slice that gets there), so both CTAs of
// a pair agree.
template <class G>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(256, 1)
flep_gemm2_slice(const __grid_constant__ Gemm2Args g, uint32_t gx, uint32_t gy, uint32_t offset, const SliceParams sp) {
  __shared__ uint32_t s_go;
  if (threadIdx.x == 0) {
    uint32_t* dp = sp.decision + sp.slice;
    uint32_t d = ld_relaxed_gpu(dp);
    bool go;
    if ((d >> 2) == slice_tag(sp.gen)) {
      go = (d & 3u) == kSliceRun;
    } else if ((d & 3u) == kSliceRun) {
      go = false;
    } else {
      const uint32_t c = ld_relaxed_gpu(sp.ctrl);
      const bool stop = ctrl_gen(c) == (sp.gen & kCtrlGenMask) && ctrl_n(c) > 0;
      const uint32_t want = (slice_tag(sp.gen) << 2) | (stop ? kSliceSkip : kSliceRun);
      const uint32_t old = atomicCAS(dp, d, want);
      go = ((old == d) ? want : old) == ((slice_tag(sp.gen) << 2) | kSliceRun);
    }
    s_go = go ? 1u : 0u;
  }
  __syncthreads();
  if (!s_go) return;                   // both CTAs of the pair leave (same decision)
  G::setup();
  const uint32_t b = offset + (blockIdx.x >> 1);
  bool given = false;
  G::pipeline(g, gx, gy, [&](uint32_t& b0, uint32_t& b1) {
    if (given) return false;
    given = true; b0 = b; b1 = b + 1;
    return true;
  });
  G::teardown();
}

// Static persistent twin (U1): the same pairs, tiles pair, pair + P, pair + 2P, ... with no
// counter and no poll (the FLEP worker's overhead baseline).
template <class G>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(256, 1)
flep_gemm2_static(const __grid_constant__ Gemm2Args g, uint32_t gx, uint32_t gy, uint32_t n_tiles) {
  G::setup();
  const uint32_t pair = blockIdx.x >> 1, pairs = gridDim.x >> 1;
  uint32_t next = pair;
  G::pipeline(g, gx, gy, [&](uint32_t& b0, uint32_t& b1) {
    if (next >= n_tiles) return false;
    b0 = next; b1 = next + 1; next += pairs;
    return true;
  });
  G::teardown();
}


}  // namespace flep
