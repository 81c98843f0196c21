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
// Preemption granularity: one tile (the pair polls between chunks; no in-tile spill here, the
// 1-CTA GEMM body keeps that). A spatial request releases a pair iff it names either of its SMs
// (a pair cannot split), R32.
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
  __nv_bfloat16* c;            // C [M,N] bf16 row-major
  uint32_t m, n, k;
};

struct Gemm2 {
  static constexpr int kThreads = 256;
  static constexpr uint32_t BM = 128, BN = 256, BK = 64, UMMA_K = 16, STAGES = 6;
  static constexpr uint32_t TM = 2 * BM;                       // tile rows of the pair
  static constexpr uint32_t kBytesA = BM * BK * 2, kBytesB = (BN / 2) * BK * 2, kStage = kBytesA + kBytesB;
  static constexpr uint32_t kTmemCols = 512;                   // two 128-lane x 256-column accumulators
  static constexpr uint32_t QDEPTH = 4;
  static constexpr uint32_t kQConsumers = 10;                  // leader: MMA + 4 epilogue warps; peer: producer + 4
  static constexpr size_t kDynSmem = 1024 + STAGES * kStage + 1024;
  static constexpr uint32_t STOP = 0xffffffffu;

  struct State {
    uint64_t full[STAGES], empty[STAGES];
    uint64_t tfull[2], tempty[2];
    uint64_t qfull[QDEPTH], qempty[QDEPTH];
    uint32_t tile_q[QDEPTH];
    uint32_t tmem_base;
    uint32_t smid;
  };

  __device__ static uint8_t* ring() {
    extern __shared__ uint8_t dsmem[];
    const uint32_t a = static_cast<uint32_t>(__cvta_generic_to_shared(dsmem));
    return dsmem + (((a + 1023u) & ~1023u) - a);
  }
  __device__ static State* state() { return reinterpret_cast<State*>(ring() + STAGES * kStage); }
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
  static constexpr uint32_t kIdesc = (1u << 4) | (1u << 7) | (1u << 10) | ((BN >> 3) << 17) | ((TM >> 4) << 24);

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
          tma_2sm(&g.tma_b, sa + kBytesA, fb, (int32_t)(kb * BK), tn * (int32_t)BN + (int32_t)(r * (BN / 2)));
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
        wait(&s->tempty[acc], aph ^ 1u);                 // both CTAs' epilogues drained this half
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint32_t tmem = tmem0 + acc * BN;
        for (uint32_t kb = 0; kb < nk; ++kb) {
          wait(&s->full[st], ph);
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          const uint32_t sa = su32(base + st * kStage), sb = sa + kBytesA;
#pragma unroll
          for (uint32_t k = 0; k < BK / UMMA_K; ++k) {
            const uint64_t da = sdesc(sa + k * UMMA_K * 2), db = sdesc(sb + k * UMMA_K * 2);
            const uint32_t accum = (kb | k) ? 1u : 0u;
            asm volatile(
                "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
                " tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n}\n"
                :: "r"(tmem), "l"(da), "l"(db), "r"(kIdesc), "r"(accum) : "memory");
          }
          // frees stage st in both CTAs
          asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                       :: "r"(su32(&s->empty[st])), "h"((uint16_t)3) : "memory");
          if (++st == STAGES) { st = 0; ph ^= 1u; }
        }
        // the accumulator half is complete in both CTAs' TMEM
        asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                     :: "r"(su32(&s->tfull[acc])), "h"((uint16_t)3) : "memory");
        if (++acc == 2) { acc = 0; aph ^= 1u; }
      }
    } else if (warp >= 4) {                              // ---- epilogue: this CTA's 128 rows
      const uint32_t q = warp - 4;
      const uint32_t rl = q * 32u + lane;
      uint32_t qi = 0, qph = 0, acc = 0, aph = 0;
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
        const uint32_t row = (uint32_t)tm * TM + r * BM + rl;
        __nv_bfloat16* crow = g.c + (size_t)row * g.n + (size_t)tn * BN;
#pragma unroll 1
        for (uint32_t c0 = 0; c0 < BN; c0 += 32) {
          uint32_t v[32];
          GemmBody::tmem_ld32(tmem + c0, v);
          uint4 o[4];
          uint32_t* ow = reinterpret_cast<uint32_t*>(o);
#pragma unroll
          for (int i = 0; i < 16; ++i) {
            __nv_bfloat162 h = __floats2bfloat162_rn(__uint_as_float(v[2 * i]), __uint_as_float(v[2 * i + 1]));
            ow[i] = *reinterpret_cast<uint32_t*>(&h);
          }
          uint4* dst = reinterpret_cast<uint4*>(crow + c0);
#pragma unroll
          for (int i = 0; i < 4; ++i) dst[i] = o[i];
        }
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncwarp();
        if (lane == 0) {
          if (leader) arrive_local(&s->tempty[acc]);
          else arrive_remote(tempty0 + acc * 8u);
        }
        if (++acc == 2) { acc = 0; aph ^= 1u; }
      }
    }
  }
};

// Worker (the PAIR is the FLEP worker: wid = cluster index, W = pairs). The leader runs the
// scheduling step of flep_worker (next_chunk: poll every K chunks, fetch C tiles, exit event);
// the spatial check uses the pair's lower-ranked SM so that a request naming either SM releases it.
template <bool kCoverage>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(Gemm2::kThreads, 1)
flep_gemm2_worker(const __grid_constant__ Gemm2Args g, const WorkerParams p) {
  __shared__ WorkerShared ws;
  const uint32_t wid = blockIdx.x >> 1;
  const bool leader = Gemm2::rank() == 0;
  if (threadIdx.x == 0) {
    ws.sm = smid_reg(); ws.t_entry = gtimer(); ws.blocks = 0; ws.reason = 0;
    ws.counted = 0; ws.last = 0; ws.ev_raw = 0; ws.ev_part = 0; ws.partial = 0;
    if (wid == 0 && leader && p.started_hint && p.status) st_relaxed_sys(&p.status->started, p.epoch);
  }
  Gemm2::setup();
  uint32_t yield_sm = 0;
  if (leader && threadIdx.x == 0) {                    // the pair's SM with the lower rank (spatial)
    uint32_t peer_sm;
    asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(peer_sm) : "r"(Gemm2::peer_addr(&Gemm2::state()->smid, 1)) : "memory");
    yield_sm = p.rank[peer_sm] < p.rank[ws.sm] ? peer_sm : ws.sm;
    ws.sm = yield_sm;                                  // the worker record names the deciding SM
  }
  SchedState st;
  Gemm2::pipeline(g, p.gx, p.gy, [&](uint32_t& b0, uint32_t& b1) {
    b0 = next_chunk(p, st, ws, wid, yield_sm);
    if (b0 == 0xffffffffu) return false;
    b1 = min(b0 + p.chunk, p.n_blocks);
    if (kCoverage)
      for (uint32_t b = b0; b < b1; ++b) atomicAdd(&p.cov[b], 1u);
    return true;
  });
  Gemm2::teardown();
  if (leader && threadIdx.x == 0) worker_exit(p, ws, wid);
}

// The original kernel (unwrapped twin): one pair per tile.
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(Gemm2::kThreads, 1)
flep_gemm2_unwrapped(const __grid_constant__ Gemm2Args g, uint32_t gx, uint32_t gy, uint32_t offset) {
  Gemm2::setup();
  const uint32_t b = offset + (blockIdx.x >> 1) + (gridDim.x >> 1) * blockIdx.y;
  bool given = false;
  Gemm2::pipeline(g, gx, gy, [&](uint32_t& b0, uint32_t& b1) {
    if (given) return false;
    given = true; b0 = b; b1 = b + 1;
    return true;
  });
  Gemm2::teardown();
}

// Kernel slicing with the device check (R31): one pair per tile of the slice; every CTA follows
// the slice's one decision (taken by the first CTA of the slice that gets there), so both CTAs of
// a pair agree.
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(Gemm2::kThreads, 1)
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
  Gemm2::setup();
  const uint32_t b = offset + (blockIdx.x >> 1);
  bool given = false;
  Gemm2::pipeline(g, gx, gy, [&](uint32_t& b0, uint32_t& b1) {
    if (given) return false;
    given = true; b0 = b; b1 = b + 1;
    return true;
  });
  Gemm2::teardown();
}

// Static persistent twin (U1): the same pairs, tiles pair, pair + P, pair + 2P, ... with no
// counter and no poll (the FLEP worker's overhead baseline).
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(Gemm2::kThreads, 1)
flep_gemm2_static(const __grid_constant__ Gemm2Args g, uint32_t gx, uint32_t gy, uint32_t n_tiles) {
  Gemm2::setup();
  const uint32_t pair = blockIdx.x >> 1, pairs = gridDim.x >> 1;
  uint32_t next = pair;
  Gemm2::pipeline(g, gx, gy, [&](uint32_t& b0, uint32_t& b1) {
    if (next >= n_tiles) return false;
    b0 = next; b1 = next + 1; next += pairs;
    return true;
  });
  Gemm2::teardown();
}


}  // namespace flep
