// flep_device.cuh — the preemptable persistent-CTA wrapper for sm_100a.
//
// Paper mapping (P:N = line N of the FLEP paper text):
//   persistent threads, W = num_SMs x max_CTAs_per_SM resident workers ..... P:128
//   pull_task(): global atomic task counter, one thread per CTA + smem bcast
//   temporal check at the loop top, amortised over L tasks ................. Fig. 4(a)(b)
//   spatial check hostSM_ID < spa_P (here: rank[%smid] < n) ................ Fig. 4(c)
//   progress tracked in a global counter so a relaunch resumes ............. P:126
//
// B200 design: one 32-bit control word ctrl = epoch<<8 | n in device memory (24
// generation bits, the same width as the host status word, so a late request never matches a
// later epoch of a pooled control block; n <= 255 covers the 148 SMs, n >= #SMs = temporal),
// polled with ld.acquire.gpu (an L2 hit) once per K chunks; a chunk is C original blocks per
// atomicAdd (the probe measured ~1.46 fetches/ns chip-wide on one address, so C amortises the
// atomic); exits happen only at poll points or on exhaustion, never while holding a chunk
// (exactly-once, reading A4). Exit accounting (reading R23): the counter and the exit counts share
// one 64-bit word; a worker's exit is counted by its exhausted fetch (the fetch that returns a
// value >= N, which it makes anyway), or by one yield-exit increment if it never made one, so a
// grid that runs to completion does no atomic at exit. The issuer of the W-th exit event
// records the epoch; a PREEMPTED epoch is published to a pinned host slot with one relaxed
// system-scope 8-byte store, a DONE epoch is seen by the host as the grid's completion (R24).
#pragma once
#include <cstdint>

namespace flep {

constexpr uint32_t kReasonYield = 1;
constexpr uint32_t kReasonExhausted = 2;
constexpr uint32_t kStatePreempted = 3;
constexpr uint32_t kStateDone = 5;
constexpr uint32_t kEvEpochs = 8;       // event log ring: last 8 epochs per launch
constexpr uint32_t kNoTrigger = 0xffffffffu;

// The control word (reading R2): generation in bits 8-31 (24 bits, as in HostStatus::word), the
// yield width n in bits 0-7 (0 = no request, n >= #SMs = temporal; kCtrlAll asks every SM).
constexpr uint32_t kCtrlGenMask = 0xffffffu;
constexpr uint32_t kCtrlAll = 0xffu;
__host__ __device__ __forceinline__ uint32_t ctrl_word(uint32_t gen, uint32_t n) {
  return ((gen & kCtrlGenMask) << 8) | (n < kCtrlAll ? n : kCtrlAll);
}
__host__ __device__ __forceinline__ uint32_t ctrl_gen(uint32_t c) { return c >> 8; }
__host__ __device__ __forceinline__ uint32_t ctrl_n(uint32_t c) { return c & kCtrlAll; }

// Per-launch control block in device memory. Hot words on separate 128-B lines.
struct alignas(128) ControlBlock {
  // the counter word (R23): bits 0-31 = task counter, the next original block index to hand out
  // (D4; raw, see ctr_offset); bits 32-47 = yield exits of the current epoch; bits 48-63 =
  // original blocks those exits left unfinished in partial tile records (in-tile preemption).
  // The epoch's last worker resets the high half.
  unsigned long long cx;
  uint32_t _p0[30];
  uint32_t ctrl;           // epoch<<8 | n_yield (D1/D2, ctrl_word()); device copy for the memop transport
  uint32_t _p1[31];
  uint32_t done_gen;       // generation whose epoch completed the launch (0 = none yet); an
                           // epoch launched after that (e.g. a refill) exits without fetching
  uint32_t pub_gen;        // generation of the last published epoch (the relay CTA's exit cue, R28)
  uint32_t _p2[30];
  // per-epoch summaries (ring of kEvEpochs)
  uint64_t ep_t_trigger[kEvEpochs];
  uint64_t ep_t_end[kEvEpochs];
  uint32_t ep_trigger_block[kEvEpochs];
  uint32_t ep_done[kEvEpochs];
  uint32_t ep_ctr[kEvEpochs];
  uint32_t ep_state[kEvEpochs];
  uint32_t ep_relay[kEvEpochs];     // request-relay CTA of the epoch (R28): smid << 8 | why it left
  uint64_t ep_relay_t[kEvEpochs];   // ... and when (%globaltimer)
};
constexpr uint32_t kRelayLeftOwnSm = 1;     // a spatial request released the relay's own SM (I3)
constexpr uint32_t kRelayLeftTemporal = 2;  // it relayed a temporal request
constexpr uint32_t kRelayLeftPublished = 3; // the epoch was published

struct WorkerEvent {       // mirrors flep_worker_event
  uint32_t smid, reason, n_blocks, epoch;
  uint64_t t_entry, t_exit;
};

struct HostStatus {        // pinned, mapped; one 32-B slot per launch
  uint32_t word;           // (generation << 8) | state of the last drained epoch   } one 8-byte
  uint32_t done;           // done counter at the end of that epoch                 } store
  uint32_t ctr;            // task counter at the end of that epoch (best effort; the device
                           // copy in ControlBlock::ep_ctr is authoritative)
  uint32_t ctrl;           // FLEP_FLAG_HOST_MAPPED: the control word itself (CPU-written)
  uint64_t t_end;          // %globaltimer of the last exit (best effort)
  uint32_t started;        // generation of the newest epoch whose first worker has started
  uint32_t _pad;
};

struct WorkerParams {
  ControlBlock* cb;
  uint32_t* ctrl;          // &cb->ctrl, or a mapped host word (FLEP_FLAG_HOST_MAPPED)
  uint32_t* cov;           // per-block execution counts or nullptr
  WorkerEvent* ev;         // [kEvEpochs][W]
  HostStatus* status;      // device alias of the pinned status word
  const uint16_t* rank;    // rank[smid]
  uint32_t n_blocks;       // N
  uint32_t chunk;          // C
  uint32_t poll;           // K
  uint32_t epoch;          // 1-based epoch number of this grid
  uint32_t workers;        // W = gridDim.x of this epoch
  uint32_t num_sms;
  uint32_t gx, gy;         // original grid (x, y); z folded into the flat index
  uint32_t trigger_block;  // device self-trigger for this epoch (kNoTrigger = none)
  uint32_t trigger_n;      // its yield width
  uint32_t prefetch;       // 1: fetch chunk j+1 while chunk j runs (hides the atomic's latency;
                           //    a stopping worker still processes the prefetched chunk)
  uint32_t gen_first;      // generation of this launch's first epoch
  uint32_t async_poll;     // 1: the poll uses the control word copied one step earlier (R22);
                           //    device-memory control word only (16-B aligned line)
  uint32_t relay_block;    // blockIdx of the request-relay CTA (R28), 0xffffffff = none; the
                           // relay is not a worker (W excludes it)
  uint32_t started_hint;   // 1: worker 0 publishes "epoch started" to the host slot at entry (a
                           //    system-scope store: the kernel's completion then waits for it)
  uint32_t ctrl_sys;       // 1: `ctrl` is a CPU-written mapped host word (FLEP_FLAG_HOST_MAPPED):
                           //    polled with a system-scope load (a gpu-scope load is not
                           //    guaranteed to observe a CPU store)
  uint32_t static_sched;   // 1: the static persistent twin (U1, flep_static): worker i takes chunks
                           //    i, i + W, i + 2W, ... with no counter, no poll, no exit accounting
  void* partial;           // in-tile preemption (FLEP_KFLAG_IN_TILE, GEMM): W partial-tile records
                           // then W accumulator spill slots (layout: partial_bytes below), or nullptr
#ifdef FLEP_TRACE
  uint64_t* trace;         // diagnostics build only: [W][kTraceChunks][2] (see flep_worker)
#endif
};
#ifdef FLEP_TRACE
constexpr uint32_t kTraceChunks = 64;
constexpr uint32_t kTraceWords = 5;    // per chunk: loop top, poll decided, step returned, after the barrier, base known
#endif

// In-tile preemption state: record i belongs to worker i of every epoch of a launch.
struct PartialTile {
  uint32_t valid;          // 1: worker i of the previous epoch stopped inside tile b
  uint32_t b;              // original block (tile) in progress
  uint32_t kb;             // first k-step not yet accumulated (0: nothing accumulated)
  uint32_t b_end;          // end of the chunk the tile belongs to (tiles b+1..b_end-1 not started)
};
constexpr size_t kSpillBytes = 128u * 256u * 4u;          // one fp32 128x256 accumulator
__host__ __device__ constexpr size_t partial_header_bytes(uint32_t workers) {
  return ((size_t)workers * sizeof(PartialTile) + 1023u) & ~(size_t)1023u;
}
__host__ __device__ constexpr size_t partial_bytes(uint32_t workers) {
  return partial_header_bytes(workers) + (size_t)workers * kSpillBytes;
}

__device__ __forceinline__ uint32_t smid_reg() {
  uint32_t r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r;
}
__device__ __forceinline__ uint64_t gtimer() {
  uint64_t r; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(r)); return r;
}
__device__ __forceinline__ uint32_t ld_acquire_gpu(const uint32_t* p) {
  uint32_t v; asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v;
}
// The poll: a relaxed gpu-scope load (served by L2, never a stale L1 line). Deliberately NOT
// ld.acquire: on sm_100a an acquire load is followed by CCTL.IVALL, which would invalidate the
// SM's whole L1 at every poll and evict the bodies' cached neighbours. Nothing read after the
// poll depends on data published before the request, so no acquire ordering is needed.
__device__ __forceinline__ uint32_t ld_relaxed_gpu(const uint32_t* p) {
  uint32_t v; asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v;
}
__device__ __forceinline__ uint32_t ld_relaxed_sys(const uint32_t* p) {
  uint32_t v; asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v;
}
__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t* p) {
  uint32_t v; asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v;
}
__device__ __forceinline__ uint32_t atom_add_acqrel_gpu(uint32_t* p, uint32_t v) {
  uint32_t old; asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory"); return old;
}
__device__ __forceinline__ void red_add_release_gpu(uint32_t* p, uint32_t v) {
  asm volatile("red.release.gpu.global.add.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_release_sys(uint32_t* p, uint32_t v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_sys(uint32_t* p, uint32_t v) {
  asm volatile("st.relaxed.sys.global.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_sys_u64(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.sys.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_gpu(uint32_t* p, uint32_t v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}

// CTA-wide barrier for original block bodies: named barrier 1 over the body's kThreads threads.
// In the unwrapped grid and the plain worker that is every thread (same as __syncthreads); in the
// scheduling-warp worker (flep_worker_sw) the extra scheduling warp does not take part.
template <int kThreads>
__device__ __forceinline__ void body_sync() {
  asm volatile("bar.sync 1, %0;" :: "n"(kThreads) : "memory");
}

// Does the control word ask the worker on `sm` to leave? (Fig. 4(c))
__device__ __forceinline__ bool should_yield(uint32_t c, const WorkerParams& p, uint32_t sm) {
  const uint32_t n = ctrl_n(c);
  if (ctrl_gen(c) != (p.epoch & kCtrlGenMask) || n == 0) return false;
  return n >= p.num_sms || p.rank[sm] < n;
}
// The poll's load of the control word: device word (stream memop / relay) -> gpu scope; mapped
// host word written by the CPU -> system scope.
__device__ __forceinline__ uint32_t poll_ctrl(const WorkerParams& p) {
  return p.ctrl_sys ? ld_relaxed_sys(p.ctrl) : ld_relaxed_gpu(p.ctrl);
}
// Device-side store of a request (self-trigger test hook, relay): a plain system-scope store to a
// mapped host word, an L2 exchange for the device word.
__device__ __forceinline__ void store_ctrl(const WorkerParams& p, uint32_t v) {
  if (p.ctrl_sys) st_relaxed_sys(p.ctrl, v);
  else atomicExch(p.ctrl, v);
}

// Worker bookkeeping shared by every loop shape (kept in shared memory, written by the one
// scheduling thread).
struct alignas(16) WorkerShared {
  uint32_t poll_buf[4];    // async poll: the control word's 16-B line, copied by cp.async.cg
  uint64_t t_entry;
  uint32_t sm, blocks, reason;
  // exit accounting (R23), written by the scheduling thread when its exit event happens
  uint32_t counted;        // the exit event has happened (exhausted fetch or yield increment)
  uint32_t last;           // ... and it was the epoch's W-th: this worker publishes the epoch
  uint32_t ev_raw;         // raw counter after that event (no fetch follows the W-th event)
  uint32_t ev_part;        // blocks left unfinished in partial tile records, including this one's
  uint32_t partial;        // blocks this worker leaves unfinished in its partial tile record
#ifdef FLEP_TRACE
  uint64_t t_poll;         // diagnostics: when the scheduling step's poll decision was taken
  uint64_t t_base;         // diagnostics: when the chunk base was known (before the next prefetch)
#endif
};

// Async poll (R22): copy the control word's 16 B from L2 (cp.async.cg bypasses L1, so it never
// returns a stale line) into shared memory without a register destination: nothing waits for
// it until the next scheduling step, and no register stays live across the body.
__device__ __forceinline__ void poll_issue(WorkerShared& ws, const uint32_t* ctrl) {
  const uint32_t dst = static_cast<uint32_t>(__cvta_generic_to_shared(ws.poll_buf));
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n cp.async.commit_group;"
               :: "r"(dst), "l"(ctrl) : "memory");
}
__device__ __forceinline__ uint32_t poll_consume(const WorkerShared& ws) {
  asm volatile("cp.async.wait_all;" ::: "memory");
  return *reinterpret_cast<const volatile uint32_t*>(ws.poll_buf);
}

// The scheduling step of Fig. 4 (b)/(c), executed by ONE thread of the worker: the amortised
// poll every K chunks, then the task fetch (pull_task) — or the chunk fetched
// ahead by the previous step when prefetching. Returns the base block of the chunk to run, or
// 0xffffffff when the worker must leave (yield on request, or counter exhausted). Never returns
// "leave" while a fetched chunk is held (exactly-once, reading A4) — except with the speculative
// fetch (R34, `rec` given), which returns such a chunk through the worker's record first. Also
// fires the device self-trigger of the test/bench hooks.
struct SchedState {
  uint32_t k = 0;                    // chunk index within the current poll period
  unsigned long long held = ~0ull;   // prefetched counter word not yet handed out (raw: the
                                     // first-epoch offset is added when it is consumed, so the
                                     // atomic's round trip overlaps the body)
  bool have_seen = false;            // async poll: a copy of the control word is in flight
  bool stopping = false;             // a request named this SM; drain the held chunk
  bool first = true;                 // first step of this worker
  uint32_t snext = 0xffffffffu;      // static twin (U1): the next chunk base of this worker
};

// pull_task. In the first epoch of a launch the counter hands out blocks after the W
// static first chunks (reading R20), so the effective counter there is ctr + W*C.
__device__ __forceinline__ uint32_t ctr_offset(const WorkerParams& p) {
  return p.epoch == p.gen_first ? p.workers * p.chunk : 0u;
}
// The counter atomic as plain PTX: atomicAdd() lets nvcc emit a warp-aggregated sequence whose
// SHFL consumes the result at once, which would make a prefetching thread wait for the whole L2
// round trip right there; with atom.add the wait happens only where the value is used.
__device__ __forceinline__ unsigned long long atom_add_cx(unsigned long long* cx, unsigned long long v) {
  unsigned long long old;
  // the address carries a lane-dependent offset that is zero for the one lane that executes it
  // (the scheduling thread is lane 0): ptxas cannot prove it warp-uniform, so it emits no
  // aggregation sequence around the atomic
  uint32_t lane;
  asm volatile("mov.u32 %0, %%laneid;" : "=r"(lane));
  asm volatile("atom.relaxed.gpu.global.add.u64 %0, [%1], %2;" : "=l"(old) : "l"(cx + lane), "l"(v) : "memory");
  return old;
}
__device__ __forceinline__ unsigned long long fetch_chunk(const WorkerParams& p) {
  return atom_add_cx(&p.cb->cx, p.chunk);
}
// First raw counter value whose fetch finds no work in this epoch (R23): the counter hands out
// multiples of C from the epoch's start, which never exceeds ceil(N/C)*C (effective).
__device__ __forceinline__ uint32_t first_exhausted_raw(const WorkerParams& p) {
  const uint32_t off = ctr_offset(p);
  const uint32_t cap = ((p.n_blocks + p.chunk - 1) / p.chunk) * p.chunk;
  return cap > off ? cap - off : 0u;
}
// This worker's exit event (R23) happened with the counter word's old value `old` (the event
// added `add_lo` to the counter): exhausted fetches before it = (raw - first exhausted) / C,
// yield exits before it = bits 32-47; the event that makes W is the epoch's last.
__device__ __forceinline__ void note_exit_event(const WorkerParams& p, WorkerShared& ws,
                                                unsigned long long old, uint32_t add_lo, uint32_t own_partial) {
  const uint32_t raw = (uint32_t)old;
  const uint32_t t = first_exhausted_raw(p);
  const uint32_t exh = raw >= t ? (raw - t) / p.chunk : 0u;
  const uint32_t yields = (uint32_t)(old >> 32) & 0xffffu;
  ws.counted = 1u;
  ws.last = (exh + yields + 1u == p.workers) ? 1u : 0u;
  ws.ev_raw = raw + add_lo;
  ws.ev_part = (uint32_t)(old >> 48) + own_partial;
}

// A worker that must leave holding a fetched, unstarted chunk (speculative fetch, R34): an
// exhausted fetch is its exit event (R23); otherwise the chunk goes to the worker's record, run
// first by the worker with the same index next epoch (the chunk-rest record of R33).
__device__ __forceinline__ void return_chunk(const WorkerParams& p, WorkerShared& ws, PartialTile* rec,
                                             unsigned long long w) {
  const uint32_t b = (uint32_t)w + ctr_offset(p);
  if (b >= p.n_blocks) {
    note_exit_event(p, ws, w, p.chunk, 0u);
    ws.reason = kReasonExhausted;
  } else {
    const uint32_t e = min(b + p.chunk, p.n_blocks);
    rec->b = b; rec->kb = 0; rec->b_end = e; rec->valid = 1;
    ws.partial = e - b;                              // the epoch cannot complete (R23)
    ws.reason = kReasonYield;
  }
}

__device__ __forceinline__ uint32_t next_chunk(const WorkerParams& p, SchedState& st, WorkerShared& ws,
                                               uint32_t wid = blockIdx.x, uint32_t yield_sm = 0xffffffffu,
                                               PartialTile* rec = nullptr) {
  // the SM whose rank a spatial request is checked against (a CTA pair passes its lower-ranked SM)
  const auto my_sm = [&]() { return yield_sm != 0xffffffffu ? yield_sm : smid_reg(); };
  if (p.static_sched) {              // U1 twin: a fixed schedule, nothing shared, never preempted
    if (st.snext == 0xffffffffu) st.snext = wid * p.chunk;
    const uint32_t b = st.snext;
    st.snext += p.workers * p.chunk;
    if (b >= p.n_blocks) { ws.reason = kReasonExhausted; return 0xffffffffu; }
    ws.blocks += min(p.chunk, p.n_blocks - b);
    return b;
  }
  uint32_t base = 0xffffffffu;
  bool have = false;
  if (st.first) {
    st.first = false;
    if (p.epoch == p.gen_first) {
      // First epoch: worker i starts on the static chunk [i*C, i*C + C) (R20): no poll and no
      // atomic before the first body, so the grid starts moving data at once. A static chunk is
      // "fetched" at launch and always processed (A4); the first poll comes at the next step.
      base = wid * p.chunk;
      have = true;
    } else {
      // A later epoch: the launch may already have completed in an earlier one (a refill raced
      // with the last blocks) -> leave without touching the counter. Both loads are issued back
      // to back: one L2 round trip. The poll doubles as the entry check of a2 (Fig. 4(c)).
      const uint32_t c = poll_ctrl(p);
      const uint32_t dg = ld_relaxed_gpu(&p.cb->done_gen);
      if (dg >= p.gen_first) { ws.reason = kReasonExhausted; return 0xffffffffu; }
      if (should_yield(c, p, my_sm())) { ws.reason = kReasonYield; return 0xffffffffu; }
    }
  } else if (st.k == 0 && !st.stopping) {            // amortised poll (Fig. 4(b))
#ifndef FLEP_NO_SPEC_FETCH
    if (rec && !p.async_poll && st.held == ~0ull) {
      // speculative fetch (reading R34): the fetch and the poll are in flight together, one
      // round trip instead of two back to back; a chunk fetched by a worker that must leave is
      // not run but returned through its record (the chunk-rest record of R33), which the worker
      // with the same index runs first in the next epoch, so a request still costs one chunk
      const unsigned long long w = fetch_chunk(p);
      const uint32_t c = poll_ctrl(p);
      if (should_yield(c, p, my_sm())) {
        st.stopping = true;
        return_chunk(p, ws, rec, w);
        return 0xffffffffu;
      }
      st.held = w;                                   // consumed just below
    } else
#endif
    {
      // async poll (FLEP_KFLAG_ASYNC_POLL, reading R22): use the word loaded at the previous step,
      // so no round trip sits between two chunks; a request is then acted on one chunk later
      const uint32_t c = (p.async_poll && st.have_seen) ? poll_consume(ws) : poll_ctrl(p);
      if (should_yield(c, p, my_sm())) { st.stopping = true; ws.reason = kReasonYield; }
    }
  }
#ifdef FLEP_TRACE
  ws.t_poll = gtimer();
#endif
  if (!have) {
    unsigned long long w = ~0ull;
    if (st.held != ~0ull) {                          // a fetched chunk is always processed (A4)
      w = st.held;
      st.held = ~0ull;
    } else if (!st.stopping) {
      w = fetch_chunk(p);
    }
    if (w != ~0ull) {
      base = (uint32_t)w + ctr_offset(p);
      // an exhausted fetch is this worker's exit event (R23); nothing is fetched after it
      if (base >= p.n_blocks) { note_exit_event(p, ws, w, p.chunk, 0u); base = 0xffffffffu; ws.reason = kReasonExhausted; }
    }
  }
  if (base != 0xffffffffu && base >= p.n_blocks) { base = 0xffffffffu; ws.reason = kReasonExhausted; }
#ifdef FLEP_TRACE
  ws.t_base = gtimer();
#endif
  if (base != 0xffffffffu) {
    ws.blocks += min(p.chunk, p.n_blocks - base);
    if (p.prefetch && !st.stopping) st.held = fetch_chunk(p);   // overlaps the body
    if (p.trigger_block - base < p.chunk) {          // device self-trigger inside this chunk
      const uint32_t e = p.epoch % kEvEpochs;
      p.cb->ep_t_trigger[e] = gtimer();
      p.cb->ep_trigger_block[e] = p.trigger_block;
      store_ctrl(p, ctrl_word(p.epoch, p.trigger_n));
    }
    if (++st.k == p.poll) st.k = 0;
    if (p.async_poll && st.k == 0 && !st.stopping) {  // the next step polls: load it now
      poll_issue(ws, p.ctrl);
      st.have_seen = true;
    }
  }
  return base;
}

// Exit path (a7), run by the worker's scheduling thread after the body's last chunk. A worker
// whose exit was counted by its exhausted fetch does no atomic here;
// any other (yield, entry exit) makes its exit event now: one 64-bit increment of the yield
// count (R23). No fences: the outputs are published by kernel completion (stream order), and
// the host status is a notification (flep_sync also waits for the grid's completion event).
__device__ __forceinline__ void worker_exit(const WorkerParams& p, WorkerShared& ws, uint32_t wid = blockIdx.x) {
  const uint64_t t_exit = gtimer();
#ifndef FLEP_NO_EVLOG          // experiment knob: no per-worker record (measures its cost)
  WorkerEvent& e = p.ev[(p.epoch % kEvEpochs) * p.workers + wid];
  e.smid = ws.sm; e.reason = ws.reason; e.n_blocks = ws.blocks; e.epoch = p.epoch;
  e.t_entry = ws.t_entry; e.t_exit = t_exit;
#endif
  if (!ws.counted) {
    const unsigned long long inc = (1ull << 32) | ((unsigned long long)ws.partial << 48);
    note_exit_event(p, ws, atom_add_cx(&p.cb->cx, inc), 0u, ws.partial);
  }
  if (ws.last) {                                       // the epoch's W-th exit event
    // every worker has made its exit event: none fetches again (some may still run the chunk
    // they hold, which they complete before the grid ends, A4)
    const bool first_epoch = p.epoch == p.gen_first;
    const bool already = !first_epoch && ld_relaxed_gpu(&p.cb->done_gen) >= p.gen_first;
    const uint32_t c = ws.ev_raw + ctr_offset(p);      // effective counter (R20)
    const bool done = already || (c >= p.n_blocks && ws.ev_part == 0u);
    const uint32_t d = done ? p.n_blocks : min(c, p.n_blocks) - ws.ev_part;
    const uint32_t st = done ? kStateDone : kStatePreempted;
    const uint32_t ei = p.epoch % kEvEpochs;
    p.cb->ep_t_end[ei] = t_exit; p.cb->ep_done[ei] = d; p.cb->ep_ctr[ei] = c;
    p.cb->ep_state[ei] = st;
    p.cb->ep_t_trigger[(p.epoch + 1) % kEvEpochs] = 0;  // next epoch's trigger stamp
    st_relaxed_gpu(&p.cb->pub_gen, p.epoch);            // the relay CTA may leave (R28)
    if (done) {                                        // clean for reuse; remember completion
      p.cb->cx = 0ull;
      if (!already) p.cb->done_gen = p.epoch;
    } else {
      // progress kept, exit counts reset; later epochs fetch from the effective counter,
      // capped at ceil(N/C)*C (only reached when partial tiles remain)
      const uint32_t cap = ((p.n_blocks + p.chunk - 1) / p.chunk) * p.chunk;
      p.cb->cx = (unsigned long long)min(c, cap);
    }
    // host notification only for a PREEMPTED epoch; DONE is seen as the grid's completion
    // (a system-scope store delays the completion by a PCIe round trip, R24)
    if (p.status && !done) {
      st_relaxed_sys(&p.status->ctr, c);
      st_relaxed_sys_u64(reinterpret_cast<uint64_t*>(&p.status->word),
                         ((uint64_t)d << 32) | ((p.epoch << 8) | st));
    }
  }
}

// Request relay (reading R28): one extra CTA of the grid, not a worker, whose thread 0 polls the
// host-written request word in the pinned slot and copies each new value into the device control
// word the workers poll. A single GPU thread sees a host store in ~1 us even while copy-engine
// work is in flight, where the stream memop takes ~5 us and tens of us behind a large H2D copy
// (probes/probe8.cu). It leaves once the epoch is published (or a temporal request was relayed:
// every worker then leaves at its next poll).
__device__ __forceinline__ void request_relay(const WorkerParams& p) {
  if (threadIdx.x != 0) return;
  const uint32_t sm = smid_reg();
  uint32_t last, why = 0;
  asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(last) : "l"(&p.status->ctrl) : "memory");
  while (!why) {
    uint32_t h;
    asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(h) : "l"(&p.status->ctrl) : "memory");
    if (h != last) {
      last = h;
      atomicExch(p.ctrl, h);
      if (ctrl_gen(h) == (p.epoch & kCtrlGenMask) && ctrl_n(h) > 0) {
        // a temporal request: every worker leaves at its next poll; a spatial one that releases
        // this SM: the relay leaves it too (I3 covers every CTA of the grid; later requests still
        // arrive by the stream memop)
        if (ctrl_n(h) >= p.num_sms) why = kRelayLeftTemporal;
        else if (p.rank[sm] < ctrl_n(h)) why = kRelayLeftOwnSm;
      }
    }
    if (!why && ld_relaxed_gpu(&p.cb->pub_gen) == p.epoch) why = kRelayLeftPublished;
  }
  const uint32_t e = p.epoch % kEvEpochs;
  p.cb->ep_relay[e] = (sm << 8) | why;
  p.cb->ep_relay_t[e] = gtimer();
}

// A chunk returned through the worker's record by the previous epoch (speculative fetch, R34):
// returns its first block, kRestLeave if the entry check says leave at once (the record stays),
// or 0xffffffff if there is none (the first epoch clears the record).
constexpr uint32_t kRestLeave = 0xfffffffeu;
__device__ __forceinline__ uint32_t take_rest(const WorkerParams& p, SchedState& st, WorkerShared& ws,
                                              PartialTile* rec) {
  if (p.epoch == p.gen_first) { rec->valid = 0; return 0xffffffffu; }
  const PartialTile e = *rec;                          // written by the previous grid
  if (!e.valid) return 0xffffffffu;
  st.first = false;                                    // (the launch is not complete)
  if (should_yield(poll_ctrl(p), p, smid_reg())) {     // entry check (a2)
    ws.reason = kReasonYield;
    ws.partial = e.b_end - e.b;
    return kRestLeave;
  }
  rec->valid = 0;
  ws.blocks += e.b_end - e.b;
  return e.b;
}

// The worker. Body contract:
//   Body::kThreads               CTA size of the original kernel
//   Body::kMinBlocks             resident CTAs per SM the register budget is sized for
//   Body::Args                   POD argument struct
//   Body::setup / teardown(args) per-worker resources (e.g. TMEM), all threads
//   Body::kPersistent == false:  Body::run(args, b0, b1, gx, gy) — all threads of the CTA execute
//                                original blocks [b0, b1) (flat b = x + gx*(y + gy*z)); the
//                                wrapper broadcasts each chunk and keeps one barrier per chunk.
//   Body::kPersistent == true:   Body::persistent(args, p, ws) owns the loop (warp-specialised
//                                bodies): its scheduling thread (tid 0) calls next_chunk() and
//                                hands chunks to the other warps itself, so chunk boundaries
//                                do not drain its pipeline.
template <class Body, bool kCoverage>
__global__ void __launch_bounds__(Body::kThreads, Body::kMinBlocks)
flep_worker(const __grid_constant__ typename Body::Args args, const WorkerParams p) {
  __shared__ uint32_t s_slot[2];     // chunk base broadcast, double-buffered: 1 barrier per chunk
  __shared__ WorkerShared ws;        // worker bookkeeping kept out of registers (tid 0 only)
  const uint32_t tid = threadIdx.x;
  if (blockIdx.x == p.relay_block) { request_relay(p); return; }   // R28: not a worker
  if (tid == 0) {
    ws.sm = smid_reg(); ws.t_entry = gtimer(); ws.blocks = 0; ws.reason = 0;
    ws.counted = 0; ws.last = 0; ws.ev_raw = 0; ws.ev_part = 0; ws.partial = 0;
    if (blockIdx.x == 0 && p.started_hint && p.status) st_relaxed_sys(&p.status->started, p.epoch);
  }
  Body::setup(args);                 // per-worker resources (e.g. TMEM, mbarriers); may sync
  if constexpr (Body::kPersistent) {
    Body::persistent(args, p, ws);
  } else {
    SchedState st;
    uint32_t parity = 0;
    // speculative fetch (FLEP_KFLAG_SPEC_FETCH, reading R34): a chunk returned by the previous
    // epoch's worker with this index is run first (after the entry check)
    PartialTile* rec = p.partial ? reinterpret_cast<PartialTile*>(p.partial) + blockIdx.x : nullptr;
    uint32_t rest = 0xffffffffu;
    if (rec && tid == 0) rest = take_rest(p, st, ws, rec);
#ifdef FLEP_TRACE
    uint32_t nchunk = 0;
#endif
    while (true) {
#ifdef FLEP_TRACE
      // diagnostics: per chunk, when tid 0 reached the scheduling step (its share of the previous
      // body done), when the poll decision was taken, when the step returned (fetch done) and
      // when the chunk barrier released it (the slowest warp of the previous body)
      const uint64_t ta = (tid == 0 && p.trace) ? gtimer() : 0;
      if (tid == 0) {
        if (rest != 0xffffffffu) { s_slot[parity] = rest == kRestLeave ? 0xffffffffu : rest; rest = 0xffffffffu; }
        else s_slot[parity] = next_chunk(p, st, ws, blockIdx.x, 0xffffffffu, rec);
      }
      const uint64_t tb = (tid == 0 && p.trace) ? gtimer() : 0;
      __syncthreads();
      if (tid == 0 && p.trace && nchunk < kTraceChunks) {
        uint64_t* t = p.trace + ((size_t)blockIdx.x * kTraceChunks + nchunk) * kTraceWords;
        t[0] = ta; t[1] = ws.t_poll; t[2] = tb; t[3] = gtimer(); t[4] = ws.t_base;
      }
      ++nchunk;
#else
      if (tid == 0) {
        if (rest != 0xffffffffu) { s_slot[parity] = rest == kRestLeave ? 0xffffffffu : rest; rest = 0xffffffffu; }
        else s_slot[parity] = next_chunk(p, st, ws, blockIdx.x, 0xffffffffu, rec);
      }
      __syncthreads();
#endif
      const uint32_t b0 = s_slot[parity];
      parity ^= 1u;
      if (b0 == 0xffffffffu) break;
      const uint32_t b1 = min(b0 + p.chunk, p.n_blocks);
      Body::run(args, b0, b1, p.gx, p.gy);
      if (kCoverage && tid == 0)
        for (uint32_t b = b0; b < b1; ++b) atomicAdd(&p.cov[b], 1u);
    }
  }
  Body::teardown(args);              // release per-worker resources before leaving the SM (a7)
  if (tid == 0) worker_exit(p, ws);
}

// ---- in-chunk stop (FLEP_KFLAG_IN_CHUNK, reading R33) --------------------------------------------
// The counter worker with C > 1 blocks per fetch (the atomic, not the poll, is what a chunk
// boundary costs) and a poll between the blocks of a chunk, so that a request is acted on after
// ONE block: the worker that stops mid-chunk leaves the rest of its chunk [b, b_end) in its
// record (the chunk-rest record of R21, without an accumulator), counted in the exit word's
// partial bits (R23, the epoch cannot complete while a record is valid); the worker with the same
// index in the next epoch runs that rest before it fetches. The poll between blocks is the async
// poll of R22 (copied during the block, tested after it) and one CTA barrier carries the decision.
template <class Body, bool kCoverage>
__global__ void __launch_bounds__(Body::kThreads, Body::kMinBlocks)
flep_worker_ic(const __grid_constant__ typename Body::Args args, const WorkerParams p) {
  __shared__ uint32_t s_rng[2][2];   // chunk [b0, b1) broadcast, double-buffered
  __shared__ uint32_t s_stop[2];     // per-block stop decision, double-buffered
  __shared__ WorkerShared ws;
  constexpr uint32_t STOP = 0xffffffffu;
  const uint32_t tid = threadIdx.x;
  if (blockIdx.x == p.relay_block) { request_relay(p); return; }   // R28: not a worker
  if (tid == 0) {
    ws.sm = smid_reg(); ws.t_entry = gtimer(); ws.blocks = 0; ws.reason = 0;
    ws.counted = 0; ws.last = 0; ws.ev_raw = 0; ws.ev_part = 0; ws.partial = 0;
    if (blockIdx.x == 0 && p.started_hint && p.status) st_relaxed_sys(&p.status->started, p.epoch);
  }
  Body::setup(args);
  PartialTile* mine = reinterpret_cast<PartialTile*>(p.partial) + blockIdx.x;
  SchedState st;
  bool restore = true;
  uint32_t par = 0, spar = 0;
  while (true) {
    if (tid == 0) {
      uint32_t b0 = STOP, b1 = 0;
      bool leave = false;
      if (restore) {                                   // the rest of a chunk stopped last epoch
        restore = false;
        if (p.epoch == p.gen_first) {
          mine->valid = 0;                             // no record survives from another launch
        } else {
          const PartialTile e = *mine;                 // written by the previous grid
          if (e.valid) {
            st.first = false;                          // (the launch is not complete)
            if (should_yield(poll_ctrl(p), p, smid_reg())) {   // entry check (a2)
              ws.reason = kReasonYield;                // the record stays for a later epoch
              ws.partial = e.b_end - e.b;
              leave = true;
            } else {
              b0 = e.b; b1 = e.b_end;
              mine->valid = 0;
              ws.blocks += b1 - b0;
            }
          }
        }
      }
      if (!leave && b0 == STOP) {
        b0 = next_chunk(p, st, ws, blockIdx.x, 0xffffffffu, mine);
        b1 = b0 == STOP ? 0u : min(b0 + p.chunk, p.n_blocks);
      }
      s_rng[par][0] = leave ? STOP : b0;
      s_rng[par][1] = b1;
    }
    __syncthreads();
    const uint32_t b0 = s_rng[par][0], b1 = s_rng[par][1];
    par ^= 1u;
    if (b0 == STOP) break;
    bool stopped = false;
    for (uint32_t b = b0; b < b1; ++b) {
      const bool more = b + 1 < b1;
      // async poll (device word), tested after this block; a CPU-written mapped word is read at
      // the decision point instead (cp.async is for device memory)
      if (tid == 0 && more && !p.ctrl_sys) poll_issue(ws, p.ctrl);
      Body::run(args, b, b + 1, p.gx, p.gy);
      if (kCoverage && tid == 0) atomicAdd(&p.cov[b], 1u);
      if (more) {
        if (tid == 0) {
          const uint32_t c = p.ctrl_sys ? poll_ctrl(p) : poll_consume(ws);
          const bool stop = should_yield(c, p, smid_reg());
          s_stop[spar] = stop ? 1u : 0u;
          if (stop) {
            mine->b = b + 1; mine->kb = 0; mine->b_end = b1; mine->valid = 1;
            ws.blocks -= b1 - (b + 1);
            ws.reason = kReasonYield;
            ws.partial = b1 - (b + 1);                 // the epoch cannot complete (R23)
          }
        }
        __syncthreads();
        stopped = s_stop[spar] != 0u;
        spar ^= 1u;
        if (stopped) break;
      }
    }
    if (stopped) break;
  }
  Body::teardown(args);
  if (tid == 0) worker_exit(p, ws);
}

// ---- scheduling-warp worker (FLEP_KFLAG_SCHED_WARP, reading R26) ------------------------------
// The same protocol as flep_worker, with the scheduling step (poll, fetch, exit accounting) run by
// one extra warp instead of thread 0 of the body: the scheduler fills a two-slot ring in shared
// memory one chunk ahead and the body warps only wait on an mbarrier, so the step's serial
// instruction chain and its round trips leave the body warps' critical path. Holding one chunk
// ahead is the prefetch of reading R3 (a stopping worker still runs the chunk it holds, A4).
__device__ __forceinline__ void sw_mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile("{\n .reg .pred p;\n W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W;\n}\n"
               :: "r"(bar), "r"(parity) : "memory");
}
__device__ __forceinline__ void sw_mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(bar) : "memory");
}
template <class Body>
struct SwMinBlocks {                 // resident CTAs per SM the register budget is sized for
  static constexpr int value = (Body::kMinBlocks * Body::kThreads) / (Body::kThreads + 32) > 0
                                   ? (Body::kMinBlocks * Body::kThreads) / (Body::kThreads + 32) : 1;
};

template <class Body, bool kCoverage>
__global__ void __launch_bounds__(Body::kThreads + 32, SwMinBlocks<Body>::value)
flep_worker_sw(const __grid_constant__ typename Body::Args args, const WorkerParams p) {
  __shared__ uint32_t s_ring[2];
  __shared__ alignas(8) uint64_t s_full[2], s_empty[2];
  __shared__ WorkerShared ws;
  constexpr uint32_t kT = Body::kThreads;
  const uint32_t tid = threadIdx.x;
  const uint32_t full0 = static_cast<uint32_t>(__cvta_generic_to_shared(&s_full[0]));
  const uint32_t empty0 = static_cast<uint32_t>(__cvta_generic_to_shared(&s_empty[0]));
  if (tid == kT) {
    ws.sm = smid_reg(); ws.t_entry = gtimer(); ws.blocks = 0; ws.reason = 0;
    ws.counted = 0; ws.last = 0; ws.ev_raw = 0; ws.ev_part = 0; ws.partial = 0;
    if (blockIdx.x == 0 && p.started_hint && p.status) st_relaxed_sys(&p.status->started, p.epoch);
    for (uint32_t i = 0; i < 2; ++i) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(full0 + 8 * i) : "memory");
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(empty0 + 8 * i) : "memory");
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  Body::setup(args);
  if (tid >= kT) {
    if (tid == kT) {                 // the scheduling lane: one chunk ahead of the body warps
      SchedState st;
      for (uint32_t j = 0;; ++j) {
        const uint32_t i = j & 1u, ph = (j >> 1) & 1u;
        if (j >= 2) sw_mbar_wait(empty0 + 8 * i, ph ^ 1u);   // slot i consumed (round j-2)
        const uint32_t b = next_chunk(p, st, ws);
        s_ring[i] = b;
        sw_mbar_arrive(full0 + 8 * i);                      // release: the body warps read s_ring[i]
        if (b == 0xffffffffu) break;
      }
    }
  } else {
    for (uint32_t j = 0;; ++j) {
      const uint32_t i = j & 1u, ph = (j >> 1) & 1u;
      sw_mbar_wait(full0 + 8 * i, ph);
      const uint32_t b0 = s_ring[i];
      if (b0 == 0xffffffffu) break;
      const uint32_t b1 = min(b0 + p.chunk, p.n_blocks);
      Body::run(args, b0, b1, p.gx, p.gy);
      if (kCoverage && tid == 0)
        for (uint32_t b = b0; b < b1; ++b) atomicAdd(&p.cov[b], 1u);
      body_sync<kT>();               // every body thread is past s_ring[i] and the chunk's smem
      if (tid == 0) sw_mbar_arrive(empty0 + 8 * i);
    }
  }
  __syncthreads();
  Body::teardown(args);
  if (tid == kT) worker_exit(p, ws);
}

// ---- warp-task worker (FLEP_KFLAG_WARP_TASKS, reading R30) ---------------------------------
// For bodies whose warps never communicate (no shared memory between warps, no CTA barrier in
// run()): a task is one warp's share of an original block (task t = b * kWarpTasks + w, run by
// Body::run_warp with the 32 lanes of one warp, exactly what warp w of the original CTA computes)
// and every warp of a worker CTA is a worker of its own: its lane 0 polls, fetches and makes its
// exit event (the same scheduling step as flep_worker, with the worker index wid = CTA * warps +
// warp), the chunk base reaches the other lanes by a shuffle, and no warp ever waits for another
// at a chunk boundary. A request is seen by each warp at its own next poll, so the drain is one
// warp task (a fraction of a block) instead of the slowest warp of a whole chunk.
template <class Body, bool kCoverage>
__global__ void __launch_bounds__(Body::kThreads, Body::kMinBlocks)
flep_warp_worker(const __grid_constant__ typename Body::Args args, const WorkerParams p) {
  constexpr uint32_t kWarps = Body::kThreads / 32;
  __shared__ WorkerShared wss[kWarps];
  if (blockIdx.x == p.relay_block) { request_relay(p); return; }   // R28: not a worker
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31u;
  const uint32_t wid = blockIdx.x * kWarps + warp;
  WorkerShared& ws = wss[warp];
  if (lane == 0) {
    ws.sm = smid_reg(); ws.t_entry = gtimer(); ws.blocks = 0; ws.reason = 0;
    ws.counted = 0; ws.last = 0; ws.ev_raw = 0; ws.ev_part = 0; ws.partial = 0;
    if (wid == 0 && p.started_hint && p.status) st_relaxed_sys(&p.status->started, p.epoch);
  }
  SchedState st;                     // used by lane 0 only
  while (true) {
    uint32_t base = 0;
    if (lane == 0) base = next_chunk(p, st, ws, wid);
    base = __shfl_sync(0xffffffffu, base, 0);
    if (base == 0xffffffffu) break;
    const uint32_t end = min(base + p.chunk, p.n_blocks);
    for (uint32_t t = base; t < end; ++t) Body::run_warp(args, t, p.gx, p.gy);
    if (kCoverage && lane == 0)
      for (uint32_t t = base; t < end; ++t) atomicAdd(&p.cov[t], 1u);
  }
  if (lane == 0) worker_exit(p, ws, wid);
}

// ---- CLC task fetch (reading R25) ----------------------------------------------
// The same preemptable persistent form with the B200's cluster launch control instead of the
// global counter: the grid is the original one in chunks (ceil(N/C) CTAs, CTA i = original blocks
// [i*C, i*C + C)) and the work queue is the hardware's queue of not-yet-launched CTAs. A running CTA runs its own block, then
// asks the hardware to cancel a pending CTA (clusterlaunchcontrol.try_cancel) and runs that
// CTA's block instead, until no CTA is left. Each original block therefore runs exactly once by
// construction (launched and run by itself, or cancelled once and run by the canceller), with
// no counter and no exit accounting.
// Preemption withdraws the persistence: at a poll point a worker named by the request (temporal,
// or rank[smid] < n) stops cancelling and leaves after the block it holds (A4: a cancelled CTA's
// block is always run). The rest of the grid stays in the hardware queue, where the CTA scheduler
// serves higher-priority streams first, so the waiting kernel gets the released SMs; an LP CTA
// that the hardware still launches meanwhile runs its one block and leaves again. Resume only
// clears the request: no relaunch, and the grid's completion is the launch's completion.
__device__ __forceinline__ void clc_try_cancel(uint32_t resp, uint32_t mbar) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], 16;" :: "r"(mbar) : "memory");
  asm volatile("clusterlaunchcontrol.try_cancel.async.shared::cta.mbarrier::complete_tx::bytes.b128 [%0], [%1];"
               :: "r"(resp), "r"(mbar) : "memory");
}
// Waits for the response; returns the cancelled CTA's x index, or 0xffffffff if none was left.
__device__ __forceinline__ uint32_t clc_response(uint32_t resp, uint32_t mbar, uint32_t phase) {
  uint32_t done = 0;
  while (!done)
    asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                 : "=r"(done) : "r"(mbar), "r"(phase) : "memory");
  uint32_t ok, x;
  asm volatile("{ .reg .pred p; .reg .b128 q; ld.shared.b128 q, [%2];"
               " clusterlaunchcontrol.query_cancel.is_canceled.pred.b128 p, q; selp.u32 %0, 1, 0, p;"
               " @p clusterlaunchcontrol.query_cancel.get_first_ctaid::x.b32.b128 %1, q; }"
               : "=r"(ok), "=r"(x) : "r"(resp) : "memory");
  return ok ? x : 0xffffffffu;
}

// A body whose run() uses no shared memory and no CTA barrier (the warp-task bodies: they define
// kWarpTasks) lets the CLC worker's warps drift between blocks like the warps of separate CTAs:
// the cancel response is broadcast through an mbarrier ring instead of a CTA barrier (below).
template <class B, class = void> struct ClcRing { static constexpr bool value = false; };
template <class B> struct ClcRing<B, decltype((void)B::kWarpTasks)> {
#ifdef FLEP_NO_CLC_RING
  static constexpr bool value = false;
#else
  static constexpr bool value = true;
#endif
};

// CLC worker without a per-block CTA barrier (reading R38, flep_clc_ring): two response slots, each with a
// "full" mbarrier (one arrival: the try_cancel's complete_tx, or thread 0's plain arrive when it
// stops cancelling, with s_stop set) and an "empty" mbarrier (one arrival per warp once its lanes
// have read the slot). Thread 0 reuses a slot only after every warp released it, so a warp that
// lags a block behind still reads its own response; every warp leaves after the response that
// says "no block" (exactly-once is unchanged: a cancelled CTA's block is run by all warps of the
// canceller, each warp its share).
template <class Body, bool kCoverage>
__device__ __forceinline__ void clc_worker_ring(const typename Body::Args& args, const WorkerParams& p,
                                                WorkerShared& ws) {
  constexpr uint32_t kWarps = Body::kThreads / 32;
  __shared__ alignas(16) uint32_t s_resp[2][4];
  __shared__ alignas(8) uint64_t s_full[2], s_empty[2];
  __shared__ uint32_t s_stop[2];
  const uint32_t tid = threadIdx.x, lane = tid & 31u;
  const uint32_t full0 = static_cast<uint32_t>(__cvta_generic_to_shared(&s_full[0]));
  const uint32_t empty0 = static_cast<uint32_t>(__cvta_generic_to_shared(&s_empty[0]));
  const uint32_t resp0 = static_cast<uint32_t>(__cvta_generic_to_shared(&s_resp[0][0]));
  if (tid == 0) {
    for (uint32_t j = 0; j < 2; ++j) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(full0 + 8u * j) : "memory");
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(empty0 + 8u * j), "r"(kWarps) : "memory");
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();                   // the only CTA barrier: the ring is initialised
  Body::setup(args);
  uint32_t b = blockIdx.x, k = 0;
  bool have_seen = false;
  for (uint32_t i = 0;; ++i) {
    const uint32_t j = i & 1u, use = i >> 1;          // slot, and how often it was used before
    if (tid == 0) {
      bool stop = false;
      if (++k == p.poll) {
        k = 0;
        const uint32_t c = (p.async_poll && have_seen) ? poll_consume(ws) : poll_ctrl(p);
        stop = should_yield(c, p, smid_reg());
      }
      if (p.async_poll && !stop && k == p.poll - 1) { poll_issue(ws, p.ctrl); have_seen = true; }
      if (use > 0) {                                 // every warp has read this slot's last response
        uint32_t done = 0;
        while (!done)
          asm volatile("{ .reg .pred q; mbarrier.try_wait.parity.shared::cta.b64 q, [%1], %2; selp.u32 %0, 1, 0, q; }"
                       : "=r"(done) : "r"(empty0 + 8u * j), "r"((use - 1u) & 1u) : "memory");
      }
      s_stop[j] = stop ? 1u : 0u;
      if (!stop) clc_try_cancel(resp0 + 16u * j, full0 + 8u * j);   // overlaps the body
      else {
        ws.reason = kReasonYield;
        asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(full0 + 8u * j) : "memory");
      }
      if (p.trigger_block - b * p.chunk < p.chunk) {   // device self-trigger (test/bench hook)
        const uint32_t e = p.epoch % kEvEpochs;
        p.cb->ep_t_trigger[e] = gtimer();
        p.cb->ep_trigger_block[e] = p.trigger_block;
        store_ctrl(p, ctrl_word(p.epoch, p.trigger_n));
      }
    }
    const uint32_t b0 = b * p.chunk, b1 = min(b0 + p.chunk, p.n_blocks);
    Body::run(args, b0, b1, p.gx, p.gy);
    if (tid == 0) {
      if (kCoverage)
        for (uint32_t bb = b0; bb < b1; ++bb) atomicAdd(&p.cov[bb], 1u);
      ws.blocks += b1 - b0;
    }
    uint32_t nb = 0xffffffffu;
    {
      uint32_t done = 0;
      while (!done)
        asm volatile("{ .reg .pred q; mbarrier.try_wait.parity.shared::cta.b64 q, [%1], %2; selp.u32 %0, 1, 0, q; }"
                     : "=r"(done) : "r"(full0 + 8u * j), "r"(use & 1u) : "memory");
      if (!s_stop[j]) {
        uint32_t ok, x;
        asm volatile("{ .reg .pred q; .reg .b128 r; ld.shared.b128 r, [%2];"
                     " clusterlaunchcontrol.query_cancel.is_canceled.pred.b128 q, r; selp.u32 %0, 1, 0, q;"
                     " @q clusterlaunchcontrol.query_cancel.get_first_ctaid::x.b32.b128 %1, r; }"
                     : "=r"(ok), "=r"(x) : "r"(resp0 + 16u * j) : "memory");
        if (ok) nb = x;
      }
      __syncwarp();
      if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(empty0 + 8u * j) : "memory");
    }
    b = nb;
    if (b == 0xffffffffu) break;
  }
  Body::teardown(args);
}

template <class Body, bool kCoverage>
__global__ void __launch_bounds__(Body::kThreads, Body::kMinBlocks)
flep_clc_ring(const __grid_constant__ typename Body::Args args, const WorkerParams p) {
  __shared__ WorkerShared ws;
  if (threadIdx.x == 0) { ws.sm = smid_reg(); ws.t_entry = gtimer(); ws.blocks = 0; ws.reason = kReasonExhausted; }
  clc_worker_ring<Body, kCoverage>(args, p, ws);
  if (threadIdx.x == 0 && blockIdx.x < p.workers) {    // event log, as in flep_clc_worker
    WorkerEvent& e = p.ev[(p.epoch % kEvEpochs) * p.workers + blockIdx.x];
    e.smid = ws.sm; e.reason = ws.reason; e.n_blocks = ws.blocks; e.epoch = p.epoch;
    e.t_entry = ws.t_entry; e.t_exit = gtimer();
  }
}
// The ring form is chosen when the worker polls at every block or every other block (K <= 2): the
// barrier form then holds every warp behind thread 0's poll round trip (measured: stencil 4096²
// C = K = 1 +18 % -> +9-10 %, SpMV-vector K = 1 +6.7 % -> +3.7 %, K = 2 61.0 -> 59.1 µs); at K = 4
// the barrier form is faster (stencil 24.3 vs 24.6 µs).
#ifndef FLEP_CLC_RING_MAXK
#define FLEP_CLC_RING_MAXK 2         // the largest K that takes the ring form (build knob)
#endif
template <class Body>
__host__ __device__ constexpr bool clc_use_ring(uint32_t poll) { return ClcRing<Body>::value && poll <= FLEP_CLC_RING_MAXK; }

template <class Body, bool kCoverage>
__global__ void __launch_bounds__(Body::kThreads, Body::kMinBlocks)
flep_clc_worker(const __grid_constant__ typename Body::Args args, const WorkerParams p) {
  __shared__ alignas(16) uint32_t s_resp[4];
  __shared__ alignas(8) uint64_t s_mbar;
  __shared__ uint32_t s_next[2];     // double-buffered broadcast: one barrier per block
  __shared__ WorkerShared ws;
  const uint32_t tid = threadIdx.x;
  const uint32_t resp = static_cast<uint32_t>(__cvta_generic_to_shared(s_resp));
  const uint32_t mbar = static_cast<uint32_t>(__cvta_generic_to_shared(&s_mbar));
  if (tid == 0) {
    ws.sm = smid_reg(); ws.t_entry = gtimer(); ws.blocks = 0; ws.reason = kReasonExhausted;
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(mbar) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  Body::setup(args);
  // CTA i of the CLC grid stands for the chunk of original blocks [i*C, i*C + C) (R25); it starts
  // on its own chunk (launched by the hardware)
  uint32_t b = blockIdx.x;
  uint32_t k = 0, phase = 0, parity = 0;
  bool have_seen = false;            // async poll: a copy of the control word is in flight
  while (true) {
    bool pending = false;
    if (tid == 0) {
      // amortised poll (every K blocks) before asking for more work; a request that names this
      // SM ends the persistence after the block in hand. With FLEP_KFLAG_ASYNC_POLL (R22) the
      // word was copied into shared memory one block earlier (no round trip here; a request is
      // then seen up to one block later)
      bool stop = false;
      if (++k == p.poll) {
        k = 0;
        const uint32_t c = (p.async_poll && have_seen) ? poll_consume(ws) : poll_ctrl(p);
        stop = should_yield(c, p, smid_reg());
      }
      if (p.async_poll && !stop && k == p.poll - 1) { poll_issue(ws, p.ctrl); have_seen = true; }
      if (!stop) { clc_try_cancel(resp, mbar); pending = true; }   // overlaps the body
      else ws.reason = kReasonYield;
      if (p.trigger_block - b * p.chunk < p.chunk) {     // device self-trigger (test/bench hook)
        const uint32_t e = p.epoch % kEvEpochs;
        p.cb->ep_t_trigger[e] = gtimer();
        p.cb->ep_trigger_block[e] = p.trigger_block;
        store_ctrl(p, ctrl_word(p.epoch, p.trigger_n));
      }
    }
    const uint32_t b0 = b * p.chunk, b1 = min(b0 + p.chunk, p.n_blocks);
    Body::run(args, b0, b1, p.gx, p.gy);
    if (tid == 0) {
      if (kCoverage)
        for (uint32_t bb = b0; bb < b1; ++bb) atomicAdd(&p.cov[bb], 1u);
      ws.blocks += b1 - b0;
      uint32_t nb = 0xffffffffu;
      if (pending) { nb = clc_response(resp, mbar, phase); phase ^= 1u; }   // a cancelled CTA's chunk is always run
      s_next[parity] = nb;
    }
    __syncthreads();
    b = s_next[parity];
    parity ^= 1u;
    if (b == 0xffffffffu) break;
  }
  Body::teardown(args);
  // event log: the first W CTAs (the first wave, which does nearly all the work) record their exit
  if (tid == 0 && blockIdx.x < p.workers) {
    WorkerEvent& e = p.ev[(p.epoch % kEvEpochs) * p.workers + blockIdx.x];
    e.smid = ws.sm; e.reason = ws.reason; e.n_blocks = ws.blocks; e.epoch = p.epoch;
    e.t_entry = ws.t_entry; e.t_exit = gtimer();
  }
}

// The original kernel (unwrapped twin, K7): one CTA per original block, same body.
#ifdef FLEP_TRACE
static __device__ uint64_t* g_unwrapped_trace;   // diagnostics build only: [N][2] entry/exit
#endif
template <class Body>
__global__ void __launch_bounds__(Body::kThreads, Body::kMinBlocks)
flep_unwrapped(const __grid_constant__ typename Body::Args args, uint32_t gx, uint32_t gy, uint32_t block_offset) {
  const uint32_t b = block_offset + blockIdx.x + gx * (blockIdx.y + gy * blockIdx.z);
#ifdef FLEP_TRACE
  const uint64_t t0 = gtimer();
#endif
  Body::setup(args);
  Body::run(args, b, b + 1, gx, gy);
  Body::teardown(args);
#ifdef FLEP_TRACE
  if (g_unwrapped_trace) {
    __syncthreads();
    if (threadIdx.x == 0) { g_unwrapped_trace[2 * (size_t)b] = t0; g_unwrapped_trace[2 * (size_t)b + 1] = gtimer(); }
  }
#endif
}

// Kernel slicing with a device-side check (FLEP_POLICY_SLICE_DEVICE, the baseline of P:96 and
// P:391, reading R31): the original kernel as sub-grids of consecutive blocks, ALL enqueued on the
// stream at launch. Every CTA of slice j follows one decision for the whole slice, taken by the
// first of its CTAs that gets there: run, or skip if a preemption request for this launch is in
// force (a slice is never split). A decision word holds the deciding epoch's tag; a RUN decided
// in an earlier epoch means the slice is done, so a resume may re-enqueue slices from any lower
// bound of the progress (the words are zeroed at the launch's first epoch).
struct SliceParams {
  const uint32_t* ctrl;    // the launch's control word (device copy)
  uint32_t* decision;      // [slices]: tag << 2 | 1 (run) or 2 (skip)
  uint32_t slice;          // j
  uint32_t gen;            // epoch generation (ctrl tag)
};
constexpr uint32_t kSliceRun = 1, kSliceSkip = 2;
__host__ __device__ __forceinline__ uint32_t slice_tag(uint32_t gen) { return gen & 0x3fffffffu; }

template <class Body>
__global__ void __launch_bounds__(Body::kThreads, Body::kMinBlocks)
flep_slice(const __grid_constant__ typename Body::Args args, uint32_t gx, uint32_t gy, uint32_t block_offset,
           const SliceParams sp) {
  __shared__ uint32_t s_go;
  if (threadIdx.x == 0) {
    uint32_t* dp = sp.decision + sp.slice;
    uint32_t d = ld_relaxed_gpu(dp);
    bool go;
    if ((d >> 2) == slice_tag(sp.gen)) {
      go = (d & 3u) == kSliceRun;                 // decided in this epoch by another CTA
    } else if ((d & 3u) == kSliceRun) {
      go = false;                                 // ran in an earlier epoch
    } else {
      const uint32_t c = ld_relaxed_gpu(sp.ctrl);
      const bool stop = ctrl_gen(c) == (sp.gen & kCtrlGenMask) && ctrl_n(c) > 0;   // slicing is temporal
      const uint32_t want = (slice_tag(sp.gen) << 2) | (stop ? kSliceSkip : kSliceRun);
      const uint32_t old = atomicCAS(dp, d, want);
      go = ((old == d) ? want : old) == ((slice_tag(sp.gen) << 2) | kSliceRun);   // first CTA decides
    }
    s_go = go ? 1u : 0u;
  }
  __syncthreads();
  if (!s_go) return;
  const uint32_t b = block_offset + blockIdx.x + gx * (blockIdx.y + gy * blockIdx.z);
  Body::setup(args);
  Body::run(args, b, b + 1, gx, gy);
  Body::teardown(args);
}

// The static persistent twin (U1): W resident CTAs, CTA i runs chunks i, i + W, ...
// of C original blocks with no counter, no poll and no exit accounting: the cost of persistence
// alone, the baseline that separates it from the FLEP wrapper's own overhead.
template <class Body>
__global__ void __launch_bounds__(Body::kThreads, Body::kMinBlocks)
flep_static(const __grid_constant__ typename Body::Args args, const WorkerParams p) {
  __shared__ WorkerShared ws;
  Body::setup(args);
  if constexpr (Body::kPersistent) {
    Body::persistent(args, p, ws);
  } else {
    for (uint32_t b0 = blockIdx.x * p.chunk; b0 < p.n_blocks; b0 += gridDim.x * p.chunk) {
      Body::run(args, b0, min(b0 + p.chunk, p.n_blocks), p.gx, p.gy);
      __syncthreads();               // the next chunk reuses the body's shared memory
    }
  }
  Body::teardown(args);
}

// Bodies without per-worker resources, run through the generic per-chunk loop.
struct NoResources {
  static constexpr bool kPersistent = false;
  template <class A> __device__ static void setup(const A&) {}
  template <class A> __device__ static void teardown(const A&) {}
  template <class A> __device__ static void persistent(const A&, const WorkerParams&, WorkerShared&) {}
};

}  // namespace flep
