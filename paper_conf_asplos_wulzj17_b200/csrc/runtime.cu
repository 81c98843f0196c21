// runtime.cu — the FLEP host runtime behind include/flep.h (§8(b)).
//
// Paper mapping:
//   interception of kernel invocations, name + config + priority to the runtime ... P:112
//   CPU state machine S1 -> S2 (await decision) -> S3 (running) -> S2 on preempt ... Fig. 5
//   preempt = set the shared variable; the GPU workers see it at their next poll ... P:164
//   resume = relaunch "to finish the remaining tasks" ........................... P:126
//   online decisions on arrive / finish, HPF + SRPT with overhead ................ §5, Fig. 6
//   duration prediction (linear model) and execution logging (T_e, T_w, T_r) ..... §4.2, §5.1
//
// B200 choices: the control word lives in device memory and is written by
// cuStreamWriteValue32 on a highest-priority control stream (executed by the GPU front end, so it
// needs no SM while the victim occupies all of them; probe: ~9 us host round trip vs ~1 ms for a
// mapped-host flag polled by 1184 CTAs). Completion / drain is published by the last exiting
// worker into a pinned host slot that the host spins on.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <array>
#include <atomic>
#include <chrono>
#include <condition_variable>
#include <deque>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "../../include/flep.h"
#include "flep_device.cuh"
#include "kernels.hpp"
#include "policy.hpp"

namespace {

using namespace flep;

thread_local std::string g_err;

flep_status fail(flep_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
  return s;
}

#define CUDA_TRY(expr)                                                                        \
  do {                                                                                        \
    cudaError_t _e = (expr);                                                                  \
    if (_e != cudaSuccess)                                                                    \
      return fail(FLEP_ERR_CUDA, "%s failed: %s (%s:%d)", #expr, cudaGetErrorString(_e),      \
                  __FILE__, __LINE__);                                                        \
  } while (0)

int64_t now_ns() {
  return std::chrono::duration_cast<std::chrono::nanoseconds>(
             std::chrono::steady_clock::now().time_since_epoch())
      .count();
}

// Driver stream memory operation for the control word, resolved through the runtime (no
// link-time libcuda). Deliberately no stream WAIT operations anywhere: a front-end wait on a
// value written by a kernel of another stream can deadlock when the two streams share a
// hardware queue (observed on the B200 probe), so ordering uses events only.
typedef CUresult (*PFN_wv32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
PFN_wv32 p_write32 = nullptr;

flep_status resolve_driver() {
  if (p_write32) return FLEP_OK;
  cudaDriverEntryPointQueryResult q;
  CUDA_TRY(cudaGetDriverEntryPoint("cuStreamWriteValue32", (void**)&p_write32, cudaEnableDefault, &q));
  if (q != cudaDriverEntryPointSuccess || !p_write32)
    return fail(FLEP_ERR_UNSUPPORTED, "cuStreamWriteValue32 not available");
  return FLEP_OK;
}

constexpr uint32_t kMaxSlots = 1u << 14;       // pinned status slots (recycled)
constexpr uint32_t kMaxSlices = 4096;          // R31: decision words per launch
constexpr uint32_t kMaxWorkersPerSm = 64;     // warp workers: 8 CTAs x 8 warps

struct Launch {
  int64_t id = 0;
  int32_t kernel = -1;
  int32_t body = 0;
  const BodyOps* ops = nullptr;
  std::vector<uint8_t> args;
  dim3 grid;
  uint32_t n_blocks = 0;
  int32_t prio = 0;
  cudaStream_t user = nullptr;
  cudaStream_t exec = nullptr;
  int exec_level = 0;
  uint32_t chunk = 1, poll = 1, workers = 0, flags = 0;
  int64_t sms_need = 0;              // SMs that host all its workers (A9), the spatial HPF input
  void* dmem = nullptr;              // ControlBlock + event ring
  ControlBlock* cb = nullptr;
  WorkerEvent* ev = nullptr;
  uint32_t* cov = nullptr;
  size_t cov_cap = 0;
  void* partial = nullptr;           // in-tile preemption records + spill slots (GEMM)
  size_t partial_cap = 0;
  int slot = -1;
  HostStatus* hs = nullptr;          // host view
  HostStatus* ds = nullptr;          // device alias
  uint32_t epoch = 0;
  int32_t state = FLEP_STATE_QUEUED;
  uint32_t n_yield = 0;
  uint32_t trig_block = kNoTrigger, trig_n = 0;
  int64_t t_arrive = 0, t_first_start = -1, t_finish = -1;
  int64_t t_e = 0, overhead = 0;
  uint32_t last_done = 0, last_ctr = 0;
  bool ctr_known = false;            // last_ctr is current (a silent DONE epoch leaves it on the device)
  int64_t t_last_request = -1, t_last_drain = -1;
  uint32_t gen0 = 0;                 // control-block generation before this launch's epoch 1
  // kernel-slicing baseline (FLEP_POLICY_SLICE): the original kernel as sub-grids of
  // slice_blocks blocks, at most two in flight; a preemption stops issuing
  bool sliced = false;
  bool slice_dev = false;            // FLEP_POLICY_SLICE_DEVICE: all slices enqueued, device check (R31)
  uint32_t* slice_dec = nullptr;     // per-slice decision words (in the control block's allocation)
  uint32_t n_slices = 0;
  bool clc = false;                  // FLEP_KFLAG_CLC: hardware work queue, resume = clear (R25)
  bool sw = false;                   // FLEP_KFLAG_SCHED_WARP: scheduling-warp worker (R26)
  bool relay = false;                // FLEP_KFLAG_HOST_RELAY: one request-relay CTA (R28)
  bool warp = false;                 // FLEP_KFLAG_WARP_TASKS: warp workers, counts in tasks (R30)
  bool ic = false;                   // FLEP_KFLAG_IN_CHUNK: poll between the blocks of a chunk (R33)
  uint32_t tasks_per_block = 1;
  uint32_t ctas = 0;                 // worker CTAs per epoch (= workers, or workers / warps per CTA)
  uint32_t slice_blocks = 0;
  uint64_t next_block = 0, slice_done = 0;
  std::deque<std::pair<cudaEvent_t, uint32_t>> inflight;
  std::vector<cudaEvent_t> evpool;
  cudaEvent_t fin_ev = nullptr;      // recorded after every grid of this launch (its last work)
  int64_t t_seen = 0;                // monitor: host time its status word was seen to move
  bool released = false;
  bool cancelled = false;
  bool materialized = false;         // device resources taken (at the first epoch, see materialize)
  bool want_cov = false;
  cudaEvent_t ev_user = nullptr;     // the caller's stream position at flep_launch (workers wait on it)
};

struct KernelReg {
  std::string name;
  int32_t body;
  uint32_t chunk, poll;
  double model[5];
  int64_t overhead;
  uint32_t flags;
  uint32_t ctas_per_sm;
};

}  // namespace

struct flep_rt_s {
  int device = 0;
  flep_options opt{};
  uint32_t num_sms = 0, nsmid = 0;
  int prio_lo = 0, prio_hi = 0;            // CUDA stream priority range (lo = least)
  cudaStream_t ctl = nullptr;              // highest-priority control stream
  cudaStream_t aux = nullptr;              // debug copies of launches whose stream went back to the pool
  uint16_t* d_rank = nullptr;
  char* cb_slab = nullptr;           // the warm control-block pool, one allocation
  size_t cb_slab_bytes = 0;
  bool in_slab(const void* p) const {
    return cb_slab && (const char*)p >= cb_slab && (const char*)p < cb_slab + cb_slab_bytes;
  }
  HostStatus* h_slots = nullptr;
  HostStatus* d_slots = nullptr;
  std::vector<int> free_slots;
  std::vector<std::pair<void*, size_t>> free_partial;
  uint64_t* trace = nullptr;        // FLEP_TRACE diagnostics builds: worker chunk trace buffer
  size_t dmem_bytes = 0;
  uint32_t max_workers = 0;
  std::vector<void*> free_dmem;
  std::map<void*, uint32_t> cb_gen;   // next free generation of each control block
  std::vector<std::pair<uint32_t*, size_t>> free_cov;
  std::map<int, std::vector<cudaStream_t>> free_streams;
  std::vector<cudaStream_t> all_streams;
  std::vector<KernelReg> kernels;
  std::map<int64_t, std::unique_ptr<Launch>> launches;
  int64_t next_id = 1;
  uint32_t arm_block = kNoTrigger, arm_n = 0;
  std::mutex mu;
  std::condition_variable cv;
  // managed mode
  std::unique_ptr<Policy> policy;
  size_t applied = 0;
  std::vector<std::array<int64_t, 7>> evlog;    // (t, type, id, prio, t_e, overhead, sms_need)
  std::thread monitor;
  std::atomic<bool> stop{false};
  std::map<std::pair<int32_t, bool>, int> occ_cache;
  std::vector<int64_t> retained;   // finished launches whose logs are kept for debug copies
  std::vector<cudaEvent_t> event_pool;
  std::vector<int64_t> to_release; // managed mode: DONE launches whose last grid may still run
  std::atomic<int> waiters{0};      // API threads waiting for `mu`
  std::vector<int64_t> active_ids;  // managed mode: launches whose state the monitor must poll
  std::atomic<uint64_t> active_gen{0};   // bumped whenever active_ids grows (wakes the monitor)
  int64_t mon_t_hit = 0, mon_t_locked = 0;   // FLEP_DEBUG_SLOW diagnostics of the monitor's pass
};

namespace {

Launch* find(flep_rt rt, flep_launch_t h);

// Lock taken by API entry points. It announces itself so the spinning monitor thread backs off
// instead of re-acquiring the (unfair) mutex immediately and starving application threads.
struct ApiLock {
  flep_rt rt;
  std::unique_lock<std::mutex> u;
  explicit ApiLock(flep_rt r) : rt(r) {
    rt->waiters.fetch_add(1, std::memory_order_relaxed);
    u = std::unique_lock<std::mutex>(rt->mu);
    rt->waiters.fetch_sub(1, std::memory_order_relaxed);
  }
};

flep_status occupancy(flep_rt rt, const BodyOps* ops, bool cov, int* k, bool sw = false, bool warp = false,
                      bool ic = false) {
  auto key = std::make_pair(ops->body * 8 + (sw ? 1 : 0) + (warp ? 2 : 0) + (ic ? 4 : 0), cov);
  auto it = rt->occ_cache.find(key);
  if (it != rt->occ_cache.end()) { *k = it->second; return FLEP_OK; }
  if (sw) CUDA_TRY(ops->occupancy_sw(k, cov));
  else if (warp) CUDA_TRY(ops->occupancy_warp(k, cov));
  else if (ic) CUDA_TRY(ops->occupancy_ic(k, cov));
  else CUDA_TRY(ops->occupancy(k, cov));
  if (*k <= 0) return fail(FLEP_ERR_UNSUPPORTED, "body %d cannot be resident", ops->body);
  rt->occ_cache[key] = *k;
  return FLEP_OK;
}

int stream_level(flep_rt rt, int32_t prio) {
  // FLEP priority (larger = higher) -> CUDA priority (numerically smaller = higher)
  int cuda_p = rt->prio_lo - (prio > 0 ? prio : 0);
  if (cuda_p < rt->prio_hi + 1) cuda_p = rt->prio_hi + 1;   // keep the top level for ctl
  if (rt->prio_hi == rt->prio_lo) cuda_p = rt->prio_lo;
  return cuda_p;
}

flep_status get_stream(flep_rt rt, int level, cudaStream_t* s) {
  auto& v = rt->free_streams[level];
  if (!v.empty()) { *s = v.back(); v.pop_back(); return FLEP_OK; }
  CUDA_TRY(cudaStreamCreateWithPriority(s, cudaStreamNonBlocking, level));
  rt->all_streams.push_back(*s);
  return FLEP_OK;
}

// Generations: every epoch of every launch that uses a control block gets a new number, so a
// late request for an old epoch (or an old launch) never matches a newer one (A2/H5).
inline uint32_t gen_of(const Launch& L) { return L.gen0 + L.epoch; }
inline uint32_t ctrl_word(const Launch& L, uint32_t n) { return flep::ctrl_word(gen_of(L), n); }

flep_status write_ctrl(flep_rt rt, Launch& L, uint32_t value) {
  L.t_last_request = now_ns();
  if (rt->opt.flag == FLEP_FLAG_HOST_MAPPED) {
    __atomic_store_n(&L.hs->ctrl, value, __ATOMIC_RELEASE);
    return FLEP_OK;
  }
  // R28: the relay CTA reads the pinned slot; written before the memop is issued, so the host
  // word is never older than the device word it feeds
  if (L.relay) __atomic_store_n(&L.hs->ctrl, value, __ATOMIC_RELEASE);
  CUresult r = p_write32((CUstream)rt->ctl, (CUdeviceptr)&L.cb->ctrl, value, 0);
  if (r != CUDA_SUCCESS) return fail(FLEP_ERR_CUDA, "cuStreamWriteValue32 failed (%d)", (int)r);
  return FLEP_OK;
}

void mark_active(flep_rt rt, Launch& L) {
  if (rt->opt.policy == FLEP_POLICY_MANUAL) return;
  if (std::find(rt->active_ids.begin(), rt->active_ids.end(), L.id) == rt->active_ids.end())
    rt->active_ids.push_back(L.id);
  rt->active_gen.fetch_add(1, std::memory_order_release);
}

flep_status pooled_event(flep_rt rt, cudaEvent_t* e) {
  if (!rt->event_pool.empty()) { *e = rt->event_pool.back(); rt->event_pool.pop_back(); return FLEP_OK; }
  CUDA_TRY(cudaEventCreateWithFlags(e, cudaEventDisableTiming));
  return FLEP_OK;
}

flep_status issue_slices(flep_rt rt, Launch& L) {
  (void)rt;
  while (L.state == FLEP_STATE_RUNNING && L.inflight.size() < 2 && L.next_block < L.n_blocks) {
    const uint32_t cnt = (uint32_t)std::min<uint64_t>(L.slice_blocks, L.n_blocks - L.next_block);
    CUDA_TRY(L.ops->unwrapped(L.args.data(), L.grid, (uint32_t)L.next_block, cnt, L.exec));
    cudaEvent_t ev;
    if (!L.evpool.empty()) { ev = L.evpool.back(); L.evpool.pop_back(); }
    else CUDA_TRY(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
    CUDA_TRY(cudaEventRecord(ev, L.exec));
    L.inflight.push_back({ev, cnt});
    L.next_block += cnt;
    CUDA_TRY(cudaEventRecord(L.fin_ev, L.exec));
  }
  return FLEP_OK;
}

// FLEP_DEBUG_SLOW=<us>: report to stderr every epoch start whose host path took longer (where the
// time went: resource materialisation vs the launch call).
int64_t slow_threshold_ns() {
  static const int64_t v = [] {
    const char* e = getenv("FLEP_DEBUG_SLOW");
    return e ? (int64_t)(atof(e) * 1e3) : (int64_t)-1;
  }();
  return v;
}

// Take the launch's device resources (first epoch only). Pools are pre-warmed so this normally
// allocates nothing.
flep_status materialize(flep_rt rt, Launch& L) {
  if (L.materialized) return FLEP_OK;
  if (rt->free_slots.empty()) return fail(FLEP_ERR_NOMEM, "out of status slots");
  flep_status s = FLEP_OK;
  int64_t tm[6] = {now_ns(), 0, 0, 0, 0, 0};
  if (L.exec_level != -1000) {
    s = get_stream(rt, L.exec_level, &L.exec);
    if (s) return s;
    tm[1] = now_ns();
    if (L.ev_user) {
      CUDA_TRY(cudaStreamWaitEvent(L.exec, L.ev_user, 0));
      rt->event_pool.push_back(L.ev_user);    // reusable once waited on (waits bind at enqueue time)
      L.ev_user = nullptr;
    }
  }
  tm[2] = now_ns();
  bool fresh_cb = false;
  if (!rt->free_dmem.empty()) { L.dmem = rt->free_dmem.back(); rt->free_dmem.pop_back(); }
  else {
    CUDA_TRY(cudaMalloc(&L.dmem, rt->dmem_bytes));
    rt->cb_gen[L.dmem] = 0;
    fresh_cb = true;             // zeroed below, on the stream the workers run on
  }
  L.gen0 = rt->cb_gen[L.dmem];
  if (L.gen0 + 2 * kEvEpochs >= kCtrlGenMask) return fail(FLEP_ERR_NOMEM, "control block generation space exhausted");
  L.cb = (ControlBlock*)L.dmem;
  L.ev = (WorkerEvent*)((char*)L.dmem + sizeof(ControlBlock));
  L.slice_dec = (uint32_t*)((char*)L.dmem + sizeof(ControlBlock) + (size_t)kEvEpochs * rt->max_workers * sizeof(WorkerEvent));
  tm[3] = now_ns();
  const uint32_t N = L.n_blocks;
  if (L.want_cov) {
    for (size_t i = 0; i < rt->free_cov.size(); ++i) {
      if (rt->free_cov[i].second >= N) {
        L.cov = rt->free_cov[i].first; L.cov_cap = rt->free_cov[i].second;
        rt->free_cov.erase(rt->free_cov.begin() + i);
        break;
      }
    }
    if (!L.cov) { L.cov_cap = std::max<size_t>(N, 4096); CUDA_TRY(cudaMalloc(&L.cov, L.cov_cap * 4)); }
  }
  if (L.flags & (FLEP_KFLAG_IN_TILE | FLEP_KFLAG_IN_CHUNK | FLEP_KFLAG_SPEC_FETCH)) {
    // per-worker partial-tile records (and, in-tile, fp32 accumulator spill slots); no reset
    // needed (the first epoch's workers clear their records)
    // (a CTA pair spills two 128-row halves: one record per pair, one slot per CTA)
    // (the wide pair tile: two slots per CTA, spill_per_cta)
    const uint32_t slots = (L.ops->max_pairs ? 2 * L.workers : L.workers) * std::max<uint32_t>(1u, L.ops->spill_per_cta);
    const size_t need = (L.flags & FLEP_KFLAG_IN_TILE) ? partial_bytes(slots) : partial_header_bytes(L.workers);
    size_t best = rt->free_partial.size();
    for (size_t i = 0; i < rt->free_partial.size(); ++i)
      if (rt->free_partial[i].second >= need &&
          (best == rt->free_partial.size() || rt->free_partial[i].second < rt->free_partial[best].second))
        best = i;
    if (best < rt->free_partial.size()) {
      L.partial = rt->free_partial[best].first; L.partial_cap = rt->free_partial[best].second;
      rt->free_partial.erase(rt->free_partial.begin() + best);
    }
    if (!L.partial) { L.partial_cap = need; CUDA_TRY(cudaMalloc(&L.partial, need)); }
  }
  L.slot = rt->free_slots.back();
  rt->free_slots.pop_back();
  L.hs = rt->h_slots + L.slot;
  L.ds = rt->d_slots + L.slot;
  memset(L.hs, 0, sizeof(HostStatus));
  // No per-launch reset work on the GPU: a pooled control block was left clean by the last
  // worker of its previous launch's DONE epoch, and its generation numbers keep increasing.
  tm[4] = now_ns();
  s = pooled_event(rt, &L.fin_ev);
  if (s) return s;
  if (L.cov) CUDA_TRY(cudaMemsetAsync(L.cov, 0, (size_t)N * 4, L.exec));
  if (fresh_cb) CUDA_TRY(cudaMemsetAsync(L.dmem, 0, sizeof(ControlBlock), L.exec));
  if (L.slice_dev) CUDA_TRY(cudaMemsetAsync(L.slice_dec, 0, (size_t)L.n_slices * 4, L.exec));   // R31
  tm[5] = now_ns();
  if (slow_threshold_ns() >= 0 && tm[5] - tm[0] > slow_threshold_ns())
    fprintf(stderr, "[flep] materialize launch %lld: stream %.1f wait %.1f block %.1f bufs %.1f event %.1f us\n",
            (long long)L.id, tm[1] ? (tm[1] - tm[0]) / 1e3 : 0.0, tm[1] ? (tm[2] - tm[1]) / 1e3 : 0.0,
            (tm[3] - tm[2]) / 1e3, (tm[4] - tm[3]) / 1e3, (tm[5] - tm[4]) / 1e3);
  L.materialized = true;
  return FLEP_OK;
}

flep_status start_epoch(flep_rt rt, Launch& L) {
  const int64_t t_a = now_ns();
  const bool fresh = !L.materialized;
  {
    flep_status s = materialize(rt, L);
    if (s) return s;
  }
  const int64_t t_b = now_ns();
  struct SlowReport {
    const Launch& L; int64_t a, b; bool fresh;
    ~SlowReport() {
      const int64_t th = slow_threshold_ns(), c = now_ns();
      if (th >= 0 && c - a > th)
        fprintf(stderr, "[flep] slow epoch start: launch %lld body %d epoch %u: materialize %.1f us%s, launch %.1f us\n",
                (long long)L.id, L.body, L.epoch, (b - a) / 1e3, fresh ? " (first)" : "", (c - b) / 1e3);
    }
  } slow_report{L, t_a, t_b, fresh};
  if (L.sliced && L.slice_dev) {
    // R31: every remaining slice goes on the stream now; each decides at its entry
    L.epoch++;
    SliceParams sp{&L.cb->ctrl, L.slice_dec, 0, gen_of(L)};
    for (uint64_t off = L.next_block; off < L.n_blocks; off += L.slice_blocks) {
      sp.slice = (uint32_t)(off / L.slice_blocks);
      const uint32_t cnt = (uint32_t)std::min<uint64_t>(L.slice_blocks, L.n_blocks - off);
      CUDA_TRY(L.ops->sliced(L.args.data(), L.grid, (uint32_t)off, cnt, sp, L.exec));
    }
    CUDA_TRY(cudaEventRecord(L.fin_ev, L.exec));
    L.state = FLEP_STATE_RUNNING;
    L.n_yield = 0;
    if (L.t_first_start < 0) L.t_first_start = now_ns();
    mark_active(rt, L);
    return FLEP_OK;
  }
  if (L.sliced) {
    L.epoch++;
    L.state = FLEP_STATE_RUNNING;
    L.n_yield = 0;
    if (L.t_first_start < 0) L.t_first_start = now_ns();
    mark_active(rt, L);
    return issue_slices(rt, L);
  }
  if (L.clc && L.epoch > 0) {        // R25: resume withdraws the request; no relaunch
    flep_status s = write_ctrl(rt, L, ctrl_word(L, 0));
    if (s) return s;
    L.state = FLEP_STATE_RUNNING;
    L.n_yield = 0;
    mark_active(rt, L);
    return FLEP_OK;
  }
  L.epoch++;
  WorkerParams p{};
  p.cb = L.cb;
  p.ctrl = rt->opt.flag == FLEP_FLAG_HOST_MAPPED ? &L.ds->ctrl : &L.cb->ctrl;
  p.cov = L.cov;
  p.ev = L.ev;
  p.status = L.ds;
  p.rank = rt->d_rank;
  p.n_blocks = L.n_blocks;
  p.chunk = L.chunk;
  p.poll = L.poll;
  p.epoch = gen_of(L);
  p.workers = L.workers;
  p.num_sms = rt->num_sms;
  p.gx = L.grid.x;
  p.gy = L.grid.y;
  p.trigger_block = L.trig_block;
  p.trigger_n = L.trig_n;
  // no prefetch with in-tile preemption: a worker whose exhausted prefetch already counted its
  // exit must not later leave a partial tile (R23)
  p.prefetch = ((L.flags & FLEP_KFLAG_PREFETCH) &&
                !(L.flags & (FLEP_KFLAG_IN_TILE | FLEP_KFLAG_IN_CHUNK | FLEP_KFLAG_SPEC_FETCH))) ? 1u : 0u;
  p.gen_first = L.gen0 + 1;
  p.started_hint = (L.flags & FLEP_KFLAG_STARTED_HINT) ? 1u : 0u;
  p.relay_block = L.relay ? L.ctas : 0xffffffffu;
  p.async_poll = ((L.flags & FLEP_KFLAG_ASYNC_POLL) && rt->opt.flag != FLEP_FLAG_HOST_MAPPED) ? 1u : 0u;
  p.ctrl_sys = rt->opt.flag == FLEP_FLAG_HOST_MAPPED ? 1u : 0u;
  p.partial = L.partial;
#ifdef FLEP_TRACE
  p.trace = rt->trace;
#endif
  L.trig_block = kNoTrigger;
  L.trig_n = 0;
  cudaError_t e = L.clc ? L.ops->clc(L.args.data(), p, (L.n_blocks + L.chunk - 1) / L.chunk, L.exec, L.cov != nullptr)
                 : L.sw ? L.ops->worker_sw(L.args.data(), p, L.workers, L.exec, L.cov != nullptr)
                 : L.warp ? L.ops->warp_worker(L.args.data(), p, L.ctas + (L.relay ? 1u : 0u), L.exec, L.cov != nullptr)
                 : L.ops->max_pairs ? L.ops->worker(L.args.data(), p, L.ctas, L.exec, L.cov != nullptr)
                 : L.ic ? L.ops->worker_ic(L.args.data(), p, L.workers + (L.relay ? 1u : 0u), L.exec, L.cov != nullptr)
                        : L.ops->worker(L.args.data(), p, L.workers + (L.relay ? 1u : 0u), L.exec, L.cov != nullptr);
  if (e != cudaSuccess) return fail(FLEP_ERR_CUDA, "worker launch failed: %s", cudaGetErrorString(e));
  CUDA_TRY(cudaEventRecord(L.fin_ev, L.exec));
  L.state = FLEP_STATE_RUNNING;
  L.n_yield = 0;
  if (L.t_first_start < 0) L.t_first_start = now_ns();
  mark_active(rt, L);
  return FLEP_OK;
}

// Pull the pinned status slot; returns true if the launch's state changed to DONE.
bool refresh(flep_rt rt, Launch& L) {
  if (L.state != FLEP_STATE_RUNNING && L.state != FLEP_STATE_YIELDING && L.state != FLEP_STATE_PARTIAL &&
      !(L.clc && L.state == FLEP_STATE_PREEMPTED))   // a preempted CLC grid still completes (R25)
    return false;
  if (L.sliced && L.slice_dev) {
    // R31: the epoch's slices have all run or been skipped once its last grid completed; the
    // skipped ones are a suffix (a request stays in force until the resume), found from the
    // decision words
    if (!(L.fin_ev && cudaEventQuery(L.fin_ev) == cudaSuccess)) return false;
    const uint32_t j0 = (uint32_t)(L.next_block / L.slice_blocks);
    std::vector<uint32_t> dec(L.n_slices - j0);
    if (!dec.empty()) {
      if (cudaMemcpyAsync(dec.data(), L.slice_dec + j0, dec.size() * 4, cudaMemcpyDeviceToHost, rt->aux) != cudaSuccess ||
          cudaStreamSynchronize(rt->aux) != cudaSuccess)
        return false;
    }
    // progress = the first slice not run in any epoch (a resume issued before this epoch's end
    // was seen starts from the older bound; its slices that already ran skip themselves)
    uint64_t next = L.n_blocks;
    for (size_t i = 0; i < dec.size(); ++i)
      if ((dec[i] & 3u) != kSliceRun) {
        next = (uint64_t)(j0 + i) * L.slice_blocks;
        break;
      }
    if (slow_threshold_ns() >= 0) {
      fprintf(stderr, "[flep] slice epoch end: launch %lld gen %u j0 %u slices %u next %llu dec:", (long long)L.id,
              gen_of(L), j0, L.n_slices, (unsigned long long)next);
      for (size_t i = 0; i < dec.size() && i < 80; ++i) fprintf(stderr, " %u:%u", dec[i] >> 2, dec[i] & 3u);
      fprintf(stderr, "\n");
    }
    L.next_block = next;
    L.slice_done = next;
    L.last_done = (uint32_t)next;
    L.last_ctr = (uint32_t)next;
    if (next >= L.n_blocks) {
      L.state = FLEP_STATE_DONE;
      L.t_finish = L.t_seen > 0 ? L.t_seen : now_ns();
      L.t_seen = 0;
      return true;
    }
    L.state = FLEP_STATE_PREEMPTED;
    L.t_last_drain = now_ns();
    return false;
  }
  if (L.sliced) {
    while (!L.inflight.empty() && cudaEventQuery(L.inflight.front().first) == cudaSuccess) {
      L.slice_done += L.inflight.front().second;
      L.evpool.push_back(L.inflight.front().first);
      L.inflight.pop_front();
    }
    if (L.state == FLEP_STATE_RUNNING) issue_slices(rt, L);
    if (!L.inflight.empty()) return false;
    L.last_done = (uint32_t)L.slice_done;
    L.last_ctr = (uint32_t)L.next_block;
    if (L.slice_done >= L.n_blocks) {
      L.state = FLEP_STATE_DONE;
      L.t_finish = now_ns();
      return true;
    }
    if (L.state == FLEP_STATE_YIELDING) { L.state = FLEP_STATE_PREEMPTED; L.t_last_drain = now_ns(); }
    return false;
  }
  // A PREEMPTED epoch is published by its last worker to the pinned slot; a DONE epoch is silent
  // on the device (a system-scope store would make the grid's completion wait for a PCIe round
  // trip, R24) and is seen as the completion of the epoch's grid. Query the grid first: once it
  // has completed, every store it made to the slot is visible, so a slot without this epoch's
  // word then means DONE.
  const bool grid_done = L.fin_ev && cudaEventQuery(L.fin_ev) == cudaSuccess;
  const uint64_t w64 = __atomic_load_n(reinterpret_cast<uint64_t*>(&L.hs->word), __ATOMIC_ACQUIRE);
  const uint32_t w = (uint32_t)w64;
  if ((w >> 8) != (gen_of(L) & 0xffffffu)) {
    if (!grid_done) return false;
    L.last_done = L.n_blocks;
    L.ctr_known = false;               // read lazily by flep_query (ControlBlock::ep_ctr)
    L.t_finish = L.t_seen > 0 ? L.t_seen : now_ns();
    L.t_seen = 0;
    L.state = FLEP_STATE_DONE;
    return true;
  }
  L.last_done = (uint32_t)(w64 >> 32);
  L.last_ctr = __atomic_load_n(&L.hs->ctr, __ATOMIC_ACQUIRE);
  L.ctr_known = true;
  // the monitor stamps the moment it saw the word move (before taking the lock)
  const int64_t t_obs = L.t_seen > 0 ? L.t_seen : now_ns();
  if (slow_threshold_ns() >= 0 && (w & 0xffu) != kStateDone)
    fprintf(stderr, "[flep] monitor: launch %lld preempted: request +0, word seen %+.3f us (%s), pass hit %+.3f, "
                    "locked %+.3f, now %+.3f\n", (long long)L.id,
            L.t_seen > 0 ? (L.t_seen - L.t_last_request) / 1e3 : -1.0, L.t_seen > 0 ? "spin" : "pass",
            (rt->mon_t_hit - L.t_last_request) / 1e3, (rt->mon_t_locked - L.t_last_request) / 1e3,
            (now_ns() - L.t_last_request) / 1e3);
  L.t_seen = 0;
  if ((w & 0xffu) == kStateDone) {
    L.state = FLEP_STATE_DONE;
    L.t_finish = t_obs;
    return true;
  }
  L.state = FLEP_STATE_PREEMPTED;
  L.t_last_drain = t_obs;
  return false;
}

// The stream a debug copy of L runs on: its own (ordered after its grids) while it has one, else
// the runtime's auxiliary stream (the stream goes back to the pool once the last grid completed).
cudaStream_t dbg_stream(flep_rt rt, const Launch& L) { return L.exec ? L.exec : rt->aux; }

// A finished launch whose last grid completed gives its execution stream back at once, even if
// its device logs are retained for debug copies.
void release_stream(flep_rt rt, Launch& L) {
  if (L.exec && L.exec_level != -1000) rt->free_streams[L.exec_level].push_back(L.exec);
  if (L.exec_level != -1000) L.exec = nullptr;
}

void release_resources(flep_rt rt, Launch& L) {
  if (L.released) return;
  // the launch's last grid has completed (caller synchronised the exec stream); the last worker
  // of the DONE epoch left the counter word at 0, so the block is reusable as is
  if (L.dmem) { rt->cb_gen[L.dmem] = gen_of(L) + 1; rt->free_dmem.push_back(L.dmem); }
  if (L.cov) rt->free_cov.push_back({L.cov, L.cov_cap});
  if (L.partial) rt->free_partial.push_back({L.partial, L.partial_cap});
  L.partial = nullptr;
  if (L.slot >= 0) rt->free_slots.push_back(L.slot);
  if (L.exec && L.exec_level != -1000) rt->free_streams[L.exec_level].push_back(L.exec);
  for (cudaEvent_t e : L.evpool) rt->event_pool.push_back(e);
  L.evpool.clear();
  if (L.ev_user) { rt->event_pool.push_back(L.ev_user); L.ev_user = nullptr; }
  if (L.fin_ev) { rt->event_pool.push_back(L.fin_ev); L.fin_ev = nullptr; }
  L.dmem = nullptr; L.cov = nullptr; L.slot = -1; L.exec = nullptr;
  L.released = true;
}

void apply_decisions(flep_rt rt) {
  const auto& d = rt->policy->decisions();
  for (; rt->applied < d.size(); ++rt->applied) {
    const Decision& x = d[rt->applied];
    auto it = rt->launches.find(x.id);
    if (it == rt->launches.end()) continue;
    Launch& L = *it->second;
    if (x.action == kPreempt) {
      const bool spatial = x.n_sms < (int64_t)rt->num_sms;
      if (L.sliced && L.slice_dev && L.state == FLEP_STATE_RUNNING) {
        // R31: the slices not yet entered skip themselves once the request is in force
        write_ctrl(rt, L, ctrl_word(L, kCtrlAll));
        L.state = FLEP_STATE_YIELDING;
        L.n_yield = (uint32_t)x.n_sms;
      } else if (L.sliced && L.state == FLEP_STATE_RUNNING) {   // slicing: stop issuing sub-kernels
        L.t_last_request = now_ns();
        L.state = FLEP_STATE_YIELDING;
        L.n_yield = (uint32_t)x.n_sms;
      } else if (L.state == FLEP_STATE_RUNNING || L.state == FLEP_STATE_PARTIAL) {
        write_ctrl(rt, L, ctrl_word(L, (uint32_t)std::min<int64_t>(x.n_sms, kCtrlAll)));
        // spatial (R29): the launch keeps running on the SMs it was not asked to release
        L.state = spatial ? FLEP_STATE_PARTIAL : FLEP_STATE_YIELDING;
        L.n_yield = (uint32_t)x.n_sms;
        if (L.clc) {                     // R25: no drain to wait for; the request is in force
          L.t_last_request = now_ns();
          L.state = spatial ? FLEP_STATE_PARTIAL : FLEP_STATE_PREEMPTED;
        }
      }
    } else if (x.action == kRefill) {
      // the guest of a spatial co-run finished: the victim goes back to every SM (f1): a CLC grid
      // just loses its request; a counter launch widens the request for its running epoch and
      // queues a full-width epoch behind it (flep_refill)
      if (L.state == FLEP_STATE_DONE) continue;       // finished meanwhile; FINISH pending
      if (L.clc) {
        write_ctrl(rt, L, ctrl_word(L, 0));
        L.state = FLEP_STATE_RUNNING;
        L.n_yield = 0;
      } else if (L.state == FLEP_STATE_PARTIAL) {
        write_ctrl(rt, L, ctrl_word(L, kCtrlAll));
        start_epoch(rt, L);
      } else if (L.state == FLEP_STATE_PREEMPTED) {
        start_epoch(rt, L);
      }
    } else {
      if (L.state == FLEP_STATE_DONE) continue;   // finished while draining; FINISH pending
      start_epoch(rt, L);
    }
  }
}

// One full pass over the active launches (caller holds rt->mu).
void monitor_pass(flep_rt rt) {
  bool changed = false;
  for (int64_t id : rt->active_ids) {
    Launch* Lp = find(rt, id);
    if (!Lp) continue;
    Launch& L = *Lp;
    if (L.state != FLEP_STATE_RUNNING && L.state != FLEP_STATE_YIELDING && L.state != FLEP_STATE_PARTIAL &&
        !(L.clc && L.state == FLEP_STATE_PREEMPTED)) continue;
    if (refresh(rt, L)) {
      rt->to_release.push_back(L.id);
      const int64_t t = L.t_finish;
      rt->evlog.push_back({t, 1, L.id, L.prio, L.t_e, L.overhead, 0});
      rt->policy->finish(t, L.id);
      apply_decisions(rt);
      changed = true;
    } else if (L.state == FLEP_STATE_PREEMPTED) {
      changed = true;
    }
  }
  if (rt->opt.policy == FLEP_POLICY_FFS) {               // FFS epochs are time-driven
    const int64_t t = now_ns();
    if (rt->policy->tick(t)) {
      rt->evlog.push_back({t, 2, -1, 0, 0, 0, 0});
      apply_decisions(rt);
      changed = true;
    }
  }
  for (size_t i = 0; i < rt->to_release.size();) {      // recycle finished launches
    Launch* R = find(rt, rt->to_release[i]);
    if (R && (!R->fin_ev || cudaEventQuery(R->fin_ev) == cudaSuccess)) {
      if (rt->opt.debug_coverage) {                    // keep the newest 64 for debug copies
        release_stream(rt, *R);
        rt->retained.push_back(R->id);
        while (rt->retained.size() > 64) {
          Launch* old = find(rt, rt->retained.front());
          rt->retained.erase(rt->retained.begin());
          if (old) release_resources(rt, *old);
        }
      } else {
        release_resources(rt, *R);
      }
      rt->to_release[i] = rt->to_release.back();
      rt->to_release.pop_back();
      changed = true;
    } else {
      ++i;
    }
  }
  // rebuild the active list
  std::vector<int64_t> keep;
  for (int64_t id : rt->active_ids) {
    Launch* L = find(rt, id);
    if (L && L->state != FLEP_STATE_DONE && L->state != FLEP_STATE_QUEUED) keep.push_back(id);
  }
  rt->active_ids.swap(keep);
  if (changed) rt->cv.notify_all();
}

// The completion monitor (a11). It polls the pinned status slots WITHOUT the runtime lock and
// takes the lock only when something changed (a status word moved, a slice or a completion event
// may have fired, an FFS epoch deadline passed), so application threads calling the API are
// never starved by it.
void monitor_loop(flep_rt rt) {
  cudaSetDevice(rt->device);
  struct Watch { const uint64_t* word; uint64_t seen; bool sliced; int64_t id; cudaEvent_t ev; bool stamped; };
  std::vector<std::pair<int64_t, int64_t>> moved;     // (launch, host time seen)
  std::vector<Watch> watch;
  int64_t deadline = -1;
  bool pending_release = false;
  uint64_t gen_seen = ~0ull;
  uint32_t spin = 0;
  bool yielding = false;             // a request is pending on some watched launch
  int64_t t_last_busy = now_ns();    // last pass with a watched launch
  while (!rt->stop.load(std::memory_order_relaxed)) {
    bool hit = false;
    if (gen_seen != rt->active_gen.load(std::memory_order_acquire)) hit = true;   // new work
    moved.clear();
    // the pinned words every pass (a plain load); the completion events of silent DONE epochs
    // (R24) every 8th pass: cudaEventQuery takes a driver lock that the application's launches
    // also need, and the PREEMPTED word is the latency-critical notification (while a request is
    // pending, every 32nd pass: a yielding launch may still end DONE, which only its event shows)
    const bool query_events = (++spin & (yielding ? 31u : 7u)) == 0;
    for (Watch& w : watch) {
      if (w.sliced) { hit = true; continue; }
      if (__atomic_load_n(w.word, __ATOMIC_ACQUIRE) != w.seen ||
          (query_events && w.ev && cudaEventQuery(w.ev) == cudaSuccess)) {
        hit = true; moved.push_back({w.id, now_ns()}); w.stamped = true;
      }
    }
    if (deadline >= 0 && now_ns() >= deadline) hit = true;
    // launches waiting for their last grid before release: checked every 64th pass only (the
    // lock is what application threads need; a release is never latency-critical)
    if (pending_release && (spin & 63u) == 0) hit = true;
    if (!hit) {
      // idle: sleep only after 50 ms without any watched launch. A sleeping monitor is woken by
      // the next flep_launch's notify, and a futex wake-up took 5-15 us: when the next launch is
      // preempted right after it starts (the bench's e2e step), the drained epoch was then seen
      // late by that much
      if (watch.empty() && deadline < 0 && now_ns() - t_last_busy > 50'000'000) {
        std::unique_lock<std::mutex> lk(rt->mu);
        rt->cv.wait_for(lk, std::chrono::milliseconds(1));
      } else {
        for (int i = 0; i < 64; ++i) __builtin_ia32_pause();
      }
      continue;
    }
    // API threads announce themselves before taking the lock (ApiLock): let them in first, for a
    // bounded time (a thread that calls the API in a loop must not starve the monitor either)
    for (int i = 0; i < 256 && rt->waiters.load(std::memory_order_relaxed) > 0; ++i) __builtin_ia32_pause();
    // while an API call holds the lock (a managed launch that preempts holds it ~10 us for its
    // driver calls), keep watching the pinned words: a drained epoch is stamped when its word
    // moves, not when the monitor gets the lock
    const int64_t t_hit = now_ns();
    std::unique_lock<std::mutex> lk(rt->mu, std::defer_lock);
    while (!lk.try_lock()) {
      for (Watch& w : watch)
        if (!w.sliced && !w.stamped && __atomic_load_n(w.word, __ATOMIC_ACQUIRE) != w.seen) {
          moved.push_back({w.id, now_ns()}); w.stamped = true;
        }
      for (int i = 0; i < 32; ++i) __builtin_ia32_pause();
    }
    rt->mon_t_hit = t_hit;
    rt->mon_t_locked = now_ns();
    for (auto& m : moved) {
      Launch* L = find(rt, m.first);
      if (L) L->t_seen = m.second;
    }
    gen_seen = rt->active_gen.load(std::memory_order_acquire);
    // snapshot the status words BEFORE the pass: a word that moves after the pass read it is
    // then seen as a change on the next poll (at worst one extra pass, never a missed event)
    std::map<int64_t, uint64_t> snap;
    for (int64_t id : rt->active_ids) {
      Launch* L = find(rt, id);
      if (L && L->hs) snap[id] = __atomic_load_n(reinterpret_cast<const uint64_t*>(&L->hs->word), __ATOMIC_ACQUIRE);
    }
    monitor_pass(rt);
    watch.clear();
    yielding = false;
    for (int64_t id : rt->active_ids) {
      Launch* L = find(rt, id);
      if (!L || !L->hs) continue;
      if (L->state == FLEP_STATE_YIELDING) yielding = true;
      const uint64_t* wp = reinterpret_cast<const uint64_t*>(&L->hs->word);
      auto it = snap.find(id);
      const bool running = L->state == FLEP_STATE_RUNNING || L->state == FLEP_STATE_YIELDING ||
                           L->state == FLEP_STATE_PARTIAL || (L->clc && L->state == FLEP_STATE_PREEMPTED);
      const bool host_sliced = L->sliced && !L->slice_dev;    // host-issued slices: every pass
      watch.push_back({wp, it != snap.end() ? it->second : ~0ull, host_sliced, id,
                       (running && !host_sliced) ? L->fin_ev : nullptr, false});
    }
    deadline = rt->policy->epoch_end();
    pending_release = !rt->to_release.empty();
    t_last_busy = now_ns();
  }
}

Launch* find(flep_rt rt, flep_launch_t h) {
  auto it = rt->launches.find(h);
  return it == rt->launches.end() ? nullptr : it->second.get();
}

flep_status validate_grid(flep_dim3 g, uint64_t* n) {
  if (g.x == 0 || g.y == 0 || g.z == 0) return fail(FLEP_ERR_INVALID, "empty grid");
  const uint64_t N = (uint64_t)g.x * g.y * g.z;
  if (N >= (1ull << 31)) return fail(FLEP_ERR_INVALID, "grid too large (%llu blocks)", (unsigned long long)N);
  *n = N;
  return FLEP_OK;
}

}  // namespace

extern "C" {

const char* flep_last_error(void) { return g_err.c_str(); }
const char* flep_version(void) { return "flep-b200 0.1 (sm_100a)"; }
int64_t flep_now_ns(void) { return now_ns(); }

flep_status flep_init(int device, const flep_options* opts, flep_rt* out) {
  if (!out) return fail(FLEP_ERR_INVALID, "out is NULL");
  *out = nullptr;
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || ndev == 0) return fail(FLEP_ERR_CUDA, "no CUDA device: %s", cudaGetErrorString(e));
  if (device < 0 || device >= ndev) return fail(FLEP_ERR_INVALID, "bad device %d", device);
  CUDA_TRY(cudaSetDevice(device));
  flep_status s = resolve_driver();
  if (s) return s;
  std::unique_ptr<flep_rt_s> rt(new flep_rt_s());
  rt->device = device;
  if (opts) rt->opt = *opts;
  if (rt->opt.default_chunk == 0) rt->opt.default_chunk = 8;
  if (rt->opt.default_poll == 0) rt->opt.default_poll = 1;
  if (rt->opt.policy < FLEP_POLICY_MANUAL || rt->opt.policy > FLEP_POLICY_SLICE_DEVICE)
    return fail(FLEP_ERR_INVALID, "bad policy %d", rt->opt.policy);
  if (rt->opt.spatial && rt->opt.policy != FLEP_POLICY_HPF)
    return fail(FLEP_ERR_INVALID, "spatial decisions need the HPF policy");
  cudaDeviceProp prop;
  CUDA_TRY(cudaGetDeviceProperties(&prop, device));
  if (prop.major != 10) return fail(FLEP_ERR_UNSUPPORTED, "needs sm_100 (got %d.%d)", prop.major, prop.minor);
  rt->num_sms = prop.multiProcessorCount;
  rt->nsmid = prop.multiProcessorCount;   // probe: %nsmid == SM count, %smid dense on B200
  CUDA_TRY(cudaDeviceGetStreamPriorityRange(&rt->prio_lo, &rt->prio_hi));
  CUDA_TRY(cudaStreamCreateWithPriority(&rt->ctl, cudaStreamNonBlocking, rt->prio_hi));
  CUDA_TRY(cudaStreamCreateWithPriority(&rt->aux, cudaStreamNonBlocking, rt->prio_lo));
  // execution streams are pre-created (4 per priority level below the control stream's): creating
  // one on the launch path costs 60 us to over 1 ms while kernels run
  for (int lv = rt->prio_lo; lv >= rt->prio_hi + 1 || (lv == rt->prio_lo && rt->prio_hi == rt->prio_lo); --lv) {
    for (int i = 0; i < 4; ++i) {
      cudaStream_t st;
      CUDA_TRY(cudaStreamCreateWithPriority(&st, cudaStreamNonBlocking, lv));
      rt->all_streams.push_back(st);
      rt->free_streams[lv].push_back(st);
    }
    if (rt->prio_hi == rt->prio_lo) break;
  }
  std::vector<uint16_t> rank(256);
  for (uint32_t i = 0; i < rank.size(); ++i) rank[i] = (uint16_t)i;
  CUDA_TRY(cudaMalloc(&rt->d_rank, rank.size() * sizeof(uint16_t)));
  CUDA_TRY(cudaMemcpy(rt->d_rank, rank.data(), rank.size() * sizeof(uint16_t), cudaMemcpyHostToDevice));
  CUDA_TRY(cudaHostAlloc(&rt->h_slots, kMaxSlots * sizeof(HostStatus), cudaHostAllocMapped));
  memset(rt->h_slots, 0, kMaxSlots * sizeof(HostStatus));
  CUDA_TRY(cudaHostGetDevicePointer(&rt->d_slots, rt->h_slots, 0));
  for (int i = kMaxSlots - 1; i >= 0; --i) rt->free_slots.push_back(i);
  rt->max_workers = rt->num_sms * kMaxWorkersPerSm;
  rt->dmem_bytes = sizeof(ControlBlock) + (size_t)kEvEpochs * rt->max_workers * sizeof(WorkerEvent) +
                  (size_t)kMaxSlices * sizeof(uint32_t);
  // warm pool: no allocation on the launch path (a managed queue holds one block per running or
  // preempted launch; nested SRPT preemptions can stack a dozen or more): 48 x ~2.4 MB carved from
  // one allocation with one memset (48 separate ones made every runtime's start ~0.2 s slower)
  {
    constexpr int kWarm = 48;
    rt->cb_slab_bytes = (size_t)kWarm * rt->dmem_bytes;
    CUDA_TRY(cudaMalloc(&rt->cb_slab, rt->cb_slab_bytes));
    CUDA_TRY(cudaMemset(rt->cb_slab, 0, rt->cb_slab_bytes));
    for (int i = 0; i < kWarm; ++i) {
      void* p = rt->cb_slab + (size_t)i * rt->dmem_bytes;
      rt->cb_gen[p] = 0;
      rt->free_dmem.push_back(p);
    }
  }
  if (rt->opt.debug_coverage) {              // debug runtimes retain 64 launches' logs: warm more
    // (coverage buffers only with bit 0)
    for (int i = 0; i < 72; ++i) {
      void* p = nullptr;
      CUDA_TRY(cudaMalloc(&p, rt->dmem_bytes));
      CUDA_TRY(cudaMemset(p, 0, sizeof(ControlBlock)));
      rt->cb_gen[p] = 0;
      rt->free_dmem.push_back(p);
      if (rt->opt.debug_coverage & 1u) {
        uint32_t* c = nullptr;
        CUDA_TRY(cudaMalloc(&c, (size_t)(1u << 20) * 4));
        rt->free_cov.push_back({c, (size_t)1u << 20});
      }
    }
  }
  if (rt->opt.policy != FLEP_POLICY_MANUAL) {
    const bool slicing = rt->opt.policy == FLEP_POLICY_SLICE || rt->opt.policy == FLEP_POLICY_SLICE_DEVICE;
    rt->policy.reset(new Policy(slicing ? (int32_t)kPolicyHPF : rt->opt.policy,
                                rt->num_sms, rt->opt.max_overhead_ppm ? rt->opt.max_overhead_ppm : 100000));
    // spatial decisions (R29): HPF on the persistent-worker mechanism only (a sliced kernel has no
    // per-SM yield)
    rt->policy->set_spatial(rt->opt.spatial != 0 && rt->opt.policy == FLEP_POLICY_HPF);
    flep_rt raw = rt.get();
    rt->monitor = std::thread([raw] { monitor_loop(raw); });
  }
  *out = rt.release();
  return FLEP_OK;
}

flep_status flep_register_body(flep_rt rt, const flep_body_ops* ops, int32_t* body_out) {
  if (!rt || !ops || !body_out) return fail(FLEP_ERR_INVALID, "NULL argument");
  const char* why = "";
  const int32_t id = register_user_body(ops, &why);
  if (id == -2) return fail(FLEP_ERR_NOMEM, "flep_register_body: %s", why);
  if (id < 0) return fail(FLEP_ERR_INVALID, "flep_register_body: %s", why);
  *body_out = id;
  return FLEP_OK;
}

flep_status flep_device_info(flep_rt rt, uint32_t* num_sms, uint32_t* nsmid) {
  if (!rt) return fail(FLEP_ERR_INVALID, "rt is NULL");
  if (num_sms) *num_sms = rt->num_sms;
  if (nsmid) *nsmid = rt->nsmid;
  return FLEP_OK;
}

flep_status flep_register_kernel(flep_rt rt, const flep_kernel_desc* d, flep_kernel* out) {
  if (!rt || !d || !out) return fail(FLEP_ERR_INVALID, "NULL argument");
  if (!body_ops(d->body)) return fail(FLEP_ERR_INVALID, "unknown body %d", d->body);
  if ((d->flags & FLEP_KFLAG_IN_TILE) && d->body != FLEP_BODY_GEMM_BF16 && d->body != FLEP_BODY_GEMM_BF16_2SM &&
      d->body != FLEP_BODY_GEMM_BF16_2SM_W)
    return fail(FLEP_ERR_UNSUPPORTED, "in-tile preemption is implemented for the GEMM bodies only");
  if ((d->flags & FLEP_KFLAG_IN_TILE) && (d->flags & FLEP_KFLAG_PREFETCH))
    return fail(FLEP_ERR_UNSUPPORTED, "in-tile preemption does not combine with chunk prefetch");
  if (d->flags & FLEP_KFLAG_IN_CHUNK) {
    const BodyOps* o = body_ops(d->body);
    if (!o->worker_ic)
      return fail(FLEP_ERR_UNSUPPORTED, "body %d has no in-chunk-stop worker", d->body);
    if (d->flags & (FLEP_KFLAG_PREFETCH | FLEP_KFLAG_CLC | FLEP_KFLAG_SCHED_WARP | FLEP_KFLAG_WARP_TASKS |
                    FLEP_KFLAG_IN_TILE))
      return fail(FLEP_ERR_UNSUPPORTED, "in-chunk stop does not combine with prefetch, CLC, the scheduling warp, "
                                        "warp tasks or in-tile preemption");
  }
  if (d->flags & FLEP_KFLAG_SPEC_FETCH) {
    if (d->body == FLEP_BODY_GEMM_BF16 || d->body == FLEP_BODY_GEMM_BF16_2SM || d->body == FLEP_BODY_GEMM_BF16_2SM_W)
      return fail(FLEP_ERR_UNSUPPORTED, "the speculative fetch is for the counter worker of the memory-bound bodies");
    // (with prefetch the next fetch would be in flight at every poll; measured slower anyway:
    // issuing it after the chunk barrier delayed the scheduling warp's own body)
    if (d->flags & (FLEP_KFLAG_PREFETCH | FLEP_KFLAG_ASYNC_POLL | FLEP_KFLAG_CLC | FLEP_KFLAG_SCHED_WARP |
                    FLEP_KFLAG_WARP_TASKS | FLEP_KFLAG_IN_TILE))
      return fail(FLEP_ERR_UNSUPPORTED, "the speculative fetch does not combine with prefetch, async poll, CLC, "
                                        "the scheduling warp, warp tasks or in-tile preemption");
  }
  ApiLock lk(rt);
  if (d->flags & FLEP_KFLAG_IN_TILE) {
    // in-tile records + accumulator spill slots for the largest worker grid this kernel can have,
    // allocated here (a cudaMalloc on the launch path took 3-50 ms while kernels ran, stalling
    // the monitor): keep three in the pool
    int kk = 0;
    flep_status s = occupancy(rt, body_ops(d->body), (rt->opt.debug_coverage & 1u) != 0, &kk);
    if (s) return s;
    if (d->ctas_per_sm && (int)d->ctas_per_sm < kk) kk = (int)d->ctas_per_sm;
    const uint32_t per_cta = std::max<uint32_t>(1u, body_ops(d->body)->spill_per_cta);
    const size_t need = partial_bytes(per_cta * std::min<uint32_t>((uint32_t)kk * rt->num_sms, rt->max_workers));
    size_t have = 0;
    for (auto& f : rt->free_partial) if (f.second >= need) ++have;
    for (; have < 3; ++have) {
      void* p = nullptr;
      CUDA_TRY(cudaMalloc(&p, need));
      rt->free_partial.push_back({p, need});
    }
  } else if (d->flags & (FLEP_KFLAG_SPEC_FETCH | FLEP_KFLAG_IN_CHUNK)) {
    // the per-worker chunk records of the speculative fetch / in-chunk stop (16 B per worker),
    // also allocated here and not on the launch path; a preempted launch keeps its buffer until
    // it completes, so a queue can hold several at once: keep eight in the pool
    int kk = 0;
    flep_status s = occupancy(rt, body_ops(d->body), (rt->opt.debug_coverage & 1u) != 0, &kk);
    if (s) return s;
    if (d->ctas_per_sm && (int)d->ctas_per_sm < kk) kk = (int)d->ctas_per_sm;
    const size_t need = partial_header_bytes(std::min<uint32_t>((uint32_t)kk * rt->num_sms, rt->max_workers));
    size_t have = 0;
    for (auto& f : rt->free_partial) if (f.second >= need) ++have;
    for (; have < 8; ++have) {
      void* p = nullptr;
      CUDA_TRY(cudaMalloc(&p, need));
      rt->free_partial.push_back({p, need});
    }
  }
  KernelReg k;
  k.name = d->name ? d->name : "";
  k.body = d->body;
  k.chunk = d->chunk ? d->chunk : rt->opt.default_chunk;
  k.poll = d->poll ? d->poll : rt->opt.default_poll;
  memcpy(k.model, d->model, sizeof(k.model));
  k.overhead = d->preempt_overhead_ns;
  k.flags = d->flags;
  k.ctas_per_sm = d->ctas_per_sm;
  rt->kernels.push_back(k);
  *out = (flep_kernel)rt->kernels.size() - 1;
  return FLEP_OK;
}

flep_status flep_workers_for(flep_rt rt, int32_t body, uint32_t* ctas_per_sm, uint32_t* workers) {
  if (!rt) return fail(FLEP_ERR_INVALID, "rt is NULL");
  const BodyOps* ops = body_ops(body);
  if (!ops) return fail(FLEP_ERR_INVALID, "unknown body %d", body);
  int k = 0;
  ApiLock lk(rt);
  flep_status s = occupancy(rt, ops, (rt->opt.debug_coverage & 1u) != 0, &k);
  if (s) return s;
  if (ctas_per_sm) *ctas_per_sm = (uint32_t)k;
  if (workers) *workers = (uint32_t)k * rt->num_sms;
  if (ops->max_pairs && workers) {                    // R32: workers are CTA pairs
    int pairs = 0;
    CUDA_TRY(ops->max_pairs(&pairs, rt->opt.debug_coverage & 1u));
    *workers = (uint32_t)pairs;
  }
  return FLEP_OK;
}

flep_status flep_launch(flep_rt rt, flep_kernel kid, flep_dim3 grid, const void* args,
                        size_t args_size, int32_t priority, flep_stream_t stream,
                        flep_launch_t* out) {
  if (!rt || !args || !out) return fail(FLEP_ERR_INVALID, "NULL argument");
  ApiLock lk(rt);
  if (kid < 0 || (size_t)kid >= rt->kernels.size()) return fail(FLEP_ERR_INVALID, "unknown kernel %d", kid);
  const KernelReg& kr = rt->kernels[kid];
  const BodyOps* ops = body_ops(kr.body);
  if (args_size != ops->args_size) return fail(FLEP_ERR_INVALID, "args_size %zu != %zu", args_size, ops->args_size);
  uint64_t N = 0;
  flep_status s = validate_grid(grid, &N);
  if (s) return s;
  dim3 g(grid.x, grid.y, grid.z);
  if (ops->validate) {
    const char* m = ops->validate(args, g);
    if (m) return fail(FLEP_ERR_INVALID, "%s", m);
  }
  const bool cov = (rt->opt.debug_coverage & 1u) != 0;
  const bool sw = (kr.flags & FLEP_KFLAG_SCHED_WARP) && !(kr.flags & FLEP_KFLAG_CLC);
  if (sw && !ops->worker_sw) return fail(FLEP_ERR_UNSUPPORTED, "body %d has no scheduling-warp worker", kr.body);
  // R30: warp tasks (not under SLICE, whose sub-kernels are the unwrapped original grid)
  const bool slicing = rt->opt.policy == FLEP_POLICY_SLICE || rt->opt.policy == FLEP_POLICY_SLICE_DEVICE;
  const bool warp = (kr.flags & FLEP_KFLAG_WARP_TASKS) && !slicing;
  if (warp && (!ops->warp_worker || !ops->warp_tasks))
    return fail(FLEP_ERR_UNSUPPORTED, "body %d has no warp-task worker", kr.body);
  if (warp && (sw || (kr.flags & (FLEP_KFLAG_CLC | FLEP_KFLAG_IN_TILE))))
    return fail(FLEP_ERR_UNSUPPORTED, "warp tasks do not combine with CLC, the scheduling warp or in-tile preemption");
  const uint32_t tpb = warp ? ops->warp_tasks : 1u;
  if (N * tpb >= (1ull << 31)) return fail(FLEP_ERR_INVALID, "grid too large for warp tasks");
  const bool ic = (kr.flags & FLEP_KFLAG_IN_CHUNK) && !slicing;
  int k = 0;
  s = occupancy(rt, ops, cov, &k, sw, warp, ic);
  if (s) return s;
  if (rt->free_slots.empty()) return fail(FLEP_ERR_NOMEM, "out of status slots");

  std::unique_ptr<Launch> Lp(new Launch());
  Launch& L = *Lp;
  L.id = rt->next_id++;
  L.kernel = kid;
  L.body = kr.body;
  L.ops = ops;
  L.args.assign((const uint8_t*)args, (const uint8_t*)args + args_size);
  L.grid = g;
  L.warp = warp;
  L.ic = ic;
  L.tasks_per_block = tpb;
  L.n_blocks = (uint32_t)(N * tpb);          // the runtime's unit: tasks (= blocks unless R30)
  L.prio = priority;
  L.user = (cudaStream_t)stream;
  L.chunk = kr.chunk;
  L.poll = kr.poll;
  L.flags = kr.flags;
  L.sw = sw;
  if (kr.flags & FLEP_KFLAG_CLC) {
    if (!ops->clc) return fail(FLEP_ERR_UNSUPPORTED, "body %d has no CLC variant", kr.body);
    if (slicing) return fail(FLEP_ERR_UNSUPPORTED, "CLC kernels cannot be sliced");
    L.clc = true;                                    // CTA i of the CLC grid = chunk i (C blocks)
  }
  if (kr.ctas_per_sm && (int)kr.ctas_per_sm < k) k = (int)kr.ctas_per_sm;
  const uint64_t wmax = (uint64_t)k * rt->num_sms;
  const uint64_t need = ((uint64_t)L.n_blocks + L.chunk - 1) / L.chunk;
  // R28: the relay CTA takes one resident slot (plain counter worker, stream-memop transport)
  L.relay = (kr.flags & FLEP_KFLAG_HOST_RELAY) && !L.sw && !L.clc && !ops->validate &&
            rt->opt.flag != FLEP_FLAG_HOST_MAPPED && wmax > 1;
  if (ops->max_pairs) {
    // R32: CTA-pair body: the worker is a cluster of 2 CTAs
    int pairs = 0;
    CUDA_TRY(ops->max_pairs(&pairs, cov));
    if (pairs <= 0) return fail(FLEP_ERR_UNSUPPORTED, "body %d: no CTA pair can be resident", kr.body);
    L.workers = (uint32_t)std::min<uint64_t>((uint64_t)pairs, need);
    L.ctas = 2 * L.workers;
    L.relay = false;
  } else if (warp) {
    // R30: worker CTAs of threads/32 warp workers each
    const uint64_t wpc = (uint64_t)ops->threads / 32u;
    const uint64_t g_need = (need + wpc - 1) / wpc;
    L.ctas = (uint32_t)std::min<uint64_t>(std::min<uint64_t>(wmax - (L.relay ? 1 : 0), g_need), rt->max_workers / wpc);
    L.workers = (uint32_t)(L.ctas * wpc);
  } else {
    L.workers = (uint32_t)std::min<uint64_t>(std::min<uint64_t>(wmax - (L.relay ? 1 : 0), need), rt->max_workers);
    L.ctas = L.workers;
  }
  {
    // SMs that host every CTA of this launch (A9: n = ceil(grid / k)): the workers
    // (+ the relay CTA), or the CLC grid's resident part
    const uint64_t ctas = L.clc ? std::min<uint64_t>(need, wmax) : (uint64_t)L.ctas + (L.relay ? 1u : 0u);
    // (a CTA-pair body: ctas = 2 x pairs, one CTA per SM)
    L.sms_need = (int64_t)std::min<uint64_t>(rt->num_sms, (ctas + (uint64_t)k - 1) / (uint64_t)k);
  }
  if (slicing) {
    L.sliced = true;                                  // R16: one slice = one wave of W*C*K blocks
    L.slice_blocks = rt->opt.slice_blocks ? rt->opt.slice_blocks
                                          : (uint32_t)std::min<uint64_t>(wmax * L.chunk * L.poll, 0x7fffffff);
    if (rt->opt.policy == FLEP_POLICY_SLICE_DEVICE) {
      if (!ops->sliced) return fail(FLEP_ERR_UNSUPPORTED, "body %d has no device-checked slice kernel", kr.body);
      L.slice_dev = true;
      // at most kMaxSlices decision words: larger slices for very large grids
      L.slice_blocks = std::max<uint32_t>(L.slice_blocks, (uint32_t)((N + kMaxSlices - 1) / kMaxSlices));
      L.n_slices = (uint32_t)((N + L.slice_blocks - 1) / L.slice_blocks);
    }
  }
  L.t_arrive = now_ns();
  L.t_e = flep_model_predict_ns(kr.model, (double)N, (double)ops->threads, (double)N, 0.0);
  L.overhead = kr.overhead;
  // the debug trigger names an original block: its first task (R30)
  L.trig_block = rt->arm_block == kNoTrigger ? kNoTrigger : rt->arm_block * tpb;
  L.trig_n = rt->arm_n;
  rt->arm_block = kNoTrigger;
  rt->arm_n = 0;
  // Device resources (control block, status slot, coverage / partial-tile buffers, execution
  // stream) are taken when the launch first runs (materialize), not at interception: a managed
  // queue can hold hundreds of intercepted launches, and only running or preempted ones need them.
  L.exec_level = stream_level(rt, priority);
  L.want_cov = cov;
  if (rt->opt.exec_on_user_stream) {
    L.exec = L.user;
    L.exec_level = -1000;
  } else {
    // the caller's prior work on `stream` (e.g. input copies) precedes the workers: its position
    // is captured now and waited on by the execution stream when the launch materialises
    s = pooled_event(rt, &L.ev_user);
    if (s) return s;
    CUDA_TRY(cudaEventRecord(L.ev_user, L.user));
  }
  rt->launches[L.id] = std::move(Lp);
  *out = L.id;
  if (rt->opt.policy == FLEP_POLICY_MANUAL) return start_epoch(rt, L);
  // managed: interception (S2) -> policy decides (Fig. 6 lines 0-15)
  rt->evlog.push_back({L.t_arrive, 0, L.id, L.prio, L.t_e, L.overhead, L.sms_need});
  rt->policy->arrive(L.t_arrive, L.id, L.prio, L.t_e, L.overhead, L.sms_need);
  apply_decisions(rt);
  rt->cv.notify_all();
  return FLEP_OK;
}

flep_status flep_preempt(flep_rt rt, flep_launch_t h, uint32_t n_sms) {
  if (!rt) return fail(FLEP_ERR_INVALID, "rt is NULL");
  if (n_sms == 0) return fail(FLEP_ERR_INVALID, "n_sms == 0");
  ApiLock lk(rt);
  if (rt->opt.policy != FLEP_POLICY_MANUAL) return fail(FLEP_ERR_STATE, "preempt is policy-driven in managed mode");
  Launch* L = find(rt, h);
  if (!L) return fail(FLEP_ERR_INVALID, "unknown launch %lld", (long long)h);
  refresh(rt, *L);
  if (L->state != FLEP_STATE_RUNNING && L->state != FLEP_STATE_PARTIAL)
    return fail(FLEP_ERR_STATE, "launch %lld is not running (state %d)", (long long)h, L->state);
  const uint32_t n = std::min<uint32_t>(n_sms, rt->num_sms);
  if (L->state == FLEP_STATE_PARTIAL && n <= L->n_yield)
    return fail(FLEP_ERR_INVALID, "a request can only widen within an epoch (%u <= %u)", n, L->n_yield);
  flep_status s = write_ctrl(rt, *L, ctrl_word(*L, n));
  if (s) return s;
  L->n_yield = n;
  L->state = n >= rt->num_sms ? FLEP_STATE_YIELDING : FLEP_STATE_PARTIAL;
  if (L->clc && n >= rt->num_sms) L->state = FLEP_STATE_PREEMPTED;   // R25: in force at once
  return FLEP_OK;
}

flep_status flep_resume(flep_rt rt, flep_launch_t h) {
  if (!rt) return fail(FLEP_ERR_INVALID, "rt is NULL");
  ApiLock lk(rt);
  if (rt->opt.policy != FLEP_POLICY_MANUAL) return fail(FLEP_ERR_STATE, "resume is policy-driven in managed mode");
  Launch* L = find(rt, h);
  if (!L) return fail(FLEP_ERR_INVALID, "unknown launch %lld", (long long)h);
  refresh(rt, *L);
  if (L->state == FLEP_STATE_PREEMPTED) return start_epoch(rt, *L);
  if (L->state == FLEP_STATE_PARTIAL) {
    flep_status s = write_ctrl(rt, *L, ctrl_word(*L, 0));
    if (s) return s;
    L->state = FLEP_STATE_RUNNING;
    L->n_yield = 0;
    return FLEP_OK;
  }
  return fail(FLEP_ERR_STATE, "launch %lld is not preempted (state %d)", (long long)h, L->state);
}

flep_status flep_refill(flep_rt rt, flep_launch_t h) {
  if (!rt) return fail(FLEP_ERR_INVALID, "rt is NULL");
  ApiLock lk(rt);
  if (rt->opt.policy != FLEP_POLICY_MANUAL) return fail(FLEP_ERR_STATE, "refill is policy-driven in managed mode");
  Launch* L = find(rt, h);
  if (!L) return fail(FLEP_ERR_INVALID, "unknown launch %lld", (long long)h);
  refresh(rt, *L);
  if (L->state == FLEP_STATE_PREEMPTED) return start_epoch(rt, *L);
  if (L->state != FLEP_STATE_PARTIAL)
    return fail(FLEP_ERR_STATE, "launch %lld is not partially preempted (state %d)", (long long)h, L->state);
  // widen the request to the whole GPU for the running epoch, then queue a full-width epoch
  // behind it (stream order): the victim is re-spread over every SM
  flep_status s = write_ctrl(rt, *L, ctrl_word(*L, kCtrlAll));
  if (s) return s;
  return start_epoch(rt, *L);
}

flep_status flep_wait_epoch(flep_rt rt, flep_launch_t h, int64_t timeout_ns) {
  if (!rt) return fail(FLEP_ERR_INVALID, "rt is NULL");
  const int64_t t0 = now_ns();
  while (true) {
    {
      ApiLock lk(rt);
      Launch* L = find(rt, h);
      if (!L) return fail(FLEP_ERR_INVALID, "unknown launch %lld", (long long)h);
      refresh(rt, *L);
      if (L->state == FLEP_STATE_PREEMPTED || L->state == FLEP_STATE_DONE || L->state == FLEP_STATE_QUEUED)
        return FLEP_OK;
    }
    if (timeout_ns >= 0 && now_ns() - t0 > timeout_ns) return fail(FLEP_ERR_TIMEOUT, "epoch did not drain");
    cudaError_t e = cudaPeekAtLastError();
    if (e != cudaSuccess) return fail(FLEP_ERR_CUDA, "sticky CUDA error: %s", cudaGetErrorString(e));
  }
}

flep_status flep_sync(flep_rt rt, flep_launch_t h, int64_t timeout_ns) {
  if (!rt) return fail(FLEP_ERR_INVALID, "rt is NULL");
  const int64_t t0 = now_ns();
  const bool managed = rt->opt.policy != FLEP_POLICY_MANUAL;
  while (true) {
    {
      ApiLock lk(rt);
      Launch* L = find(rt, h);
      if (!L) return fail(FLEP_ERR_INVALID, "unknown launch %lld", (long long)h);
      if (!managed) refresh(rt, *L);
      // DONE, and its last grid completed (queried under the lock: in managed mode the monitor
      // recycles the completion event once it has fired, so never block on it unlocked)
      if (L->state == FLEP_STATE_DONE && (L->released || !L->fin_ev || cudaEventQuery(L->fin_ev) == cudaSuccess)) break;
      if (!managed && L->state == FLEP_STATE_PREEMPTED)
        return fail(FLEP_ERR_STATE, "launch %lld is preempted; resume it first", (long long)h);
      // managed: sleep until the monitor reports a state change (no lock spinning, which would
      // starve the monitor and the other application threads)
      if (managed) rt->cv.wait_for(lk.u, std::chrono::microseconds(200));
    }
    if (timeout_ns >= 0 && now_ns() - t0 > timeout_ns) return fail(FLEP_ERR_TIMEOUT, "launch not done");
    if (!managed) std::this_thread::yield();
  }
  ApiLock lk(rt);
  Launch* L = find(rt, h);
  if (rt->opt.policy != FLEP_POLICY_MANUAL) return FLEP_OK;   // the monitor releases at DONE
  // keep the newest finished launches' device logs (coverage, events) for debug copies
  // (64 with the coverage log, else the last 4; the warm pool keeps launches allocation-free)
  const size_t kRetain = rt->opt.debug_coverage ? 64 : 4;
  if (L && !L->released && std::find(rt->retained.begin(), rt->retained.end(), h) == rt->retained.end()) {
    release_stream(rt, *L);                 // DONE and its last grid completed (checked above)
    rt->retained.push_back(h);
  }
  while (rt->retained.size() > kRetain) {
    Launch* old = find(rt, rt->retained.front());
    rt->retained.erase(rt->retained.begin());
    if (old) release_resources(rt, *old);
  }
  return FLEP_OK;
}

flep_status flep_query(flep_rt rt, flep_launch_t h, flep_launch_info* out) {
  if (!rt || !out) return fail(FLEP_ERR_INVALID, "NULL argument");
  ApiLock lk(rt);
  Launch* L = find(rt, h);
  if (!L) return fail(FLEP_ERR_INVALID, "unknown launch %lld", (long long)h);
  if (rt->opt.policy == FLEP_POLICY_MANUAL) refresh(rt, *L);
  if (L->state == FLEP_STATE_DONE && !L->ctr_known && !L->sliced && L->dmem && !L->released) {
    // the final counter of a silent DONE epoch (R24): one small copy from the control block
    uint32_t c = 0;
    const uint32_t e = gen_of(*L) % kEvEpochs;
    CUDA_TRY(cudaMemcpyAsync(&c, &L->cb->ep_ctr[e], 4, cudaMemcpyDeviceToHost, dbg_stream(rt, *L)));
    CUDA_TRY(cudaStreamSynchronize(dbg_stream(rt, *L)));
    L->last_ctr = c;
    L->ctr_known = true;
  }
  memset(out, 0, sizeof(*out));
  out->state = L->state;
  out->epoch = L->epoch;
  out->blocks_total = L->n_blocks;
  out->blocks_done = L->last_done;
  out->counter = L->last_ctr;
  out->t_arrive = L->t_arrive;
  out->t_first_start = L->t_first_start;
  out->t_finish = L->t_finish;
  out->workers = L->workers;
  out->n_yield = L->n_yield;
  out->t_e = L->t_e;
  out->t_last_request = L->t_last_request;
  out->t_last_drain = L->t_last_drain;
  if (L->hs) {
    const uint32_t g = __atomic_load_n(&L->hs->started, __ATOMIC_ACQUIRE);
    out->started_epoch = (g > L->gen0) ? g - L->gen0 : 0;
  }
  out->tasks_per_block = L->tasks_per_block;
  if (rt->policy) {
    const Policy::Entry* e = rt->policy->entry(L->id);
    if (e) { out->t_w = e->t_w; out->t_r = e->t_r; }
  }
  return FLEP_OK;
}

flep_status flep_cancel(flep_rt rt, flep_launch_t h) {
  if (!rt) return fail(FLEP_ERR_INVALID, "rt is NULL");
  const bool managed = rt->opt.policy != FLEP_POLICY_MANUAL;
  {
    ApiLock lk(rt);
    Launch* L = find(rt, h);
    if (!L) return fail(FLEP_ERR_INVALID, "unknown launch %lld", (long long)h);
    // managed modes: the monitor owns the state transitions (a DONE seen here would never reach
    // the policy); it refreshes the launch and signals the condition variable
    if (!managed) refresh(rt, *L);
    if (L->state == FLEP_STATE_DONE) return FLEP_OK;
    if (L->state == FLEP_STATE_RUNNING || L->state == FLEP_STATE_PARTIAL || L->state == FLEP_STATE_YIELDING) {
      write_ctrl(rt, *L, ctrl_word(*L, kCtrlAll));
      L->state = FLEP_STATE_YIELDING;
    }
    L->cancelled = true;
  }
  for (;;) {                               // wait for the running epoch to drain (or complete)
    ApiLock lk(rt);
    Launch* L = find(rt, h);
    if (!managed) refresh(rt, *L);
    if (L->state != FLEP_STATE_YIELDING && !(L->clc && L->state == FLEP_STATE_PREEMPTED && L->epoch > 0 &&
                                             cudaEventQuery(L->fin_ev) != cudaSuccess))
      break;
    if (managed) rt->cv.wait_for(lk.u, std::chrono::microseconds(200));
  }
  ApiLock lk(rt);
  Launch* L = find(rt, h);
  if (L->state == FLEP_STATE_DONE) return FLEP_OK;    // completed while draining (the monitor
                                                      // already told the policy, managed mode)
  if (L->exec) CUDA_TRY(cudaStreamSynchronize(L->exec));
  // the abandoned epoch left the counter word non-zero: clear the block for reuse
  if (L->epoch > 0 && L->cb && !L->sliced) {
    CUDA_TRY(cudaMemsetAsync(L->cb, 0, offsetof(ControlBlock, ep_t_trigger), dbg_stream(rt, *L)));
    CUDA_TRY(cudaStreamSynchronize(dbg_stream(rt, *L)));
  }
  L->state = FLEP_STATE_DONE;
  L->t_finish = now_ns();
  if (managed) {
    // the policy must forget it (it may think the launch runs, or hold it in a queue): a FINISH
    // event, the decisions that follow, and the launch's resources go back to the pools
    rt->evlog.push_back({L->t_finish, 1, L->id, L->prio, L->t_e, L->overhead, 0});
    rt->policy->finish(L->t_finish, L->id);
    apply_decisions(rt);
    rt->to_release.push_back(L->id);
    rt->cv.notify_all();
  }
  return FLEP_OK;
}

flep_status flep_shutdown(flep_rt rt) {
  if (!rt) return FLEP_OK;
  rt->stop = true;
  if (rt->monitor.joinable()) rt->monitor.join();
  std::vector<int64_t> ids;
  for (auto& kv : rt->launches) if (kv.second->state != FLEP_STATE_DONE) ids.push_back(kv.first);
  for (int64_t id : ids) flep_cancel(rt, id);
  cudaDeviceSynchronize();
  for (auto& kv : rt->launches) {
    Launch& L = *kv.second;
    for (cudaEvent_t e : L.evpool) cudaEventDestroy(e);
    for (auto& e : L.inflight) cudaEventDestroy(e.first);
    if (!L.released) {
      if (L.dmem && !rt->in_slab(L.dmem)) cudaFree(L.dmem);
      if (L.cov) cudaFree(L.cov);
      if (L.partial) cudaFree(L.partial);
    }
  }
  for (cudaEvent_t e : rt->event_pool) cudaEventDestroy(e);
  for (void* p : rt->free_dmem) if (!rt->in_slab(p)) cudaFree(p);
  if (rt->cb_slab) cudaFree(rt->cb_slab);
  for (auto& c : rt->free_cov) cudaFree(c.first);
  for (auto& c : rt->free_partial) cudaFree(c.first);
  for (cudaStream_t s : rt->all_streams) cudaStreamDestroy(s);
  if (rt->ctl) cudaStreamDestroy(rt->ctl);
  if (rt->aux) cudaStreamDestroy(rt->aux);
  if (rt->d_rank) cudaFree(rt->d_rank);
  if (rt->h_slots) cudaFreeHost(rt->h_slots);
  delete rt;
  return FLEP_OK;
}

flep_status flep_launch_unwrapped(flep_rt rt, int32_t body, flep_dim3 grid, const void* args,
                                  size_t args_size, flep_stream_t stream) {
  if (!rt || !args) return fail(FLEP_ERR_INVALID, "NULL argument");
  const BodyOps* ops = body_ops(body);
  if (!ops) return fail(FLEP_ERR_INVALID, "unknown body %d", body);
  if (args_size != ops->args_size) return fail(FLEP_ERR_INVALID, "args_size mismatch");
  uint64_t N = 0;
  flep_status s = validate_grid(grid, &N);
  if (s) return s;
  dim3 g(grid.x, grid.y, grid.z);
  if (ops->validate) { const char* m = ops->validate(args, g); if (m) return fail(FLEP_ERR_INVALID, "%s", m); }
  { int k; ApiLock lk(rt); s = occupancy(rt, ops, false, &k); if (s) return s; }
  CUDA_TRY(ops->unwrapped(args, g, 0, 0, (cudaStream_t)stream));
  return FLEP_OK;
}

flep_status flep_launch_static(flep_rt rt, int32_t body, flep_dim3 grid, const void* args,
                               size_t args_size, uint32_t chunk, flep_stream_t stream) {
  if (!rt || !args) return fail(FLEP_ERR_INVALID, "NULL argument");
  const BodyOps* ops = body_ops(body);
  if (!ops) return fail(FLEP_ERR_INVALID, "unknown body %d", body);
  if (!ops->static_launch) return fail(FLEP_ERR_UNSUPPORTED, "body %d has no static persistent twin", body);
  if (args_size != ops->args_size) return fail(FLEP_ERR_INVALID, "args_size mismatch");
  uint64_t N = 0;
  flep_status s = validate_grid(grid, &N);
  if (s) return s;
  dim3 g(grid.x, grid.y, grid.z);
  if (ops->validate) { const char* m = ops->validate(args, g); if (m) return fail(FLEP_ERR_INVALID, "%s", m); }
  uint32_t ctas = 0;
  {
    ApiLock lk(rt);
    int k = 0;
    s = occupancy(rt, ops, false, &k);
    if (s) return s;
    if (ops->max_pairs) {
      int pairs = 0;
      CUDA_TRY(ops->max_pairs(&pairs, false));
      ctas = 2u * (uint32_t)std::max(pairs, 1);
    } else {
      ctas = (uint32_t)k * rt->num_sms;
    }
  }
  CUDA_TRY(ops->static_launch(args, g, ctas, chunk ? chunk : 1u, (cudaStream_t)stream));
  return FLEP_OK;
}

flep_status flep_launch_sliced(flep_rt rt, int32_t body, flep_dim3 grid, const void* args,
                               size_t args_size, uint32_t slice_blocks, flep_stream_t stream) {
  if (!rt || !args) return fail(FLEP_ERR_INVALID, "NULL argument");
  if (slice_blocks == 0) return fail(FLEP_ERR_INVALID, "slice_blocks == 0");
  const BodyOps* ops = body_ops(body);
  if (!ops) return fail(FLEP_ERR_INVALID, "unknown body %d", body);
  if (args_size != ops->args_size) return fail(FLEP_ERR_INVALID, "args_size mismatch");
  uint64_t N = 0;
  flep_status s = validate_grid(grid, &N);
  if (s) return s;
  dim3 g(grid.x, grid.y, grid.z);
  if (ops->validate) { const char* m = ops->validate(args, g); if (m) return fail(FLEP_ERR_INVALID, "%s", m); }
  { int k; ApiLock lk(rt); s = occupancy(rt, ops, false, &k); if (s) return s; }
  for (uint64_t off = 0; off < N; off += slice_blocks) {
    const uint32_t cnt = (uint32_t)std::min<uint64_t>(slice_blocks, N - off);
    CUDA_TRY(ops->unwrapped(args, g, (uint32_t)off, cnt, (cudaStream_t)stream));
  }
  return FLEP_OK;
}

flep_status flep_debug_trigger_at(flep_rt rt, flep_launch_t h, uint64_t block_index, uint32_t n_sms) {
  if (!rt) return fail(FLEP_ERR_INVALID, "rt is NULL");
  ApiLock lk(rt);
  Launch* L = find(rt, h);
  if (!L) return fail(FLEP_ERR_INVALID, "unknown launch %lld", (long long)h);
  refresh(rt, *L);
  if (L->state != FLEP_STATE_PREEMPTED && L->state != FLEP_STATE_QUEUED)
    return fail(FLEP_ERR_STATE, "trigger can only be set for the next epoch of a launch that is not running");
  L->trig_block = block_index >= 0xffffffffull ? kNoTrigger : (uint32_t)(block_index * L->tasks_per_block);
  L->trig_n = std::min<uint32_t>(n_sms, kCtrlAll);
  return FLEP_OK;
}

flep_status flep_debug_arm_next_trigger(flep_rt rt, uint64_t block_index, uint32_t n_sms) {
  if (!rt) return fail(FLEP_ERR_INVALID, "rt is NULL");
  ApiLock lk(rt);
  rt->arm_block = block_index >= 0xffffffffull ? kNoTrigger : (uint32_t)block_index;
  rt->arm_n = std::min<uint32_t>(n_sms, kCtrlAll);
  return FLEP_OK;
}

flep_status flep_debug_copy_coverage(flep_rt rt, flep_launch_t h, uint32_t* host_out, size_t n) {
  if (!rt || !host_out) return fail(FLEP_ERR_INVALID, "NULL argument");
  ApiLock lk(rt);
  Launch* L = find(rt, h);
  if (!L) return fail(FLEP_ERR_INVALID, "unknown launch %lld", (long long)h);
  if (!L->cov) return fail(FLEP_ERR_STATE, "coverage log not enabled or already released");
  if (n > L->n_blocks) return fail(FLEP_ERR_INVALID, "n > N");
  CUDA_TRY(cudaMemcpyAsync(host_out, L->cov, n * 4, cudaMemcpyDeviceToHost, dbg_stream(rt, *L)));
  CUDA_TRY(cudaStreamSynchronize(dbg_stream(rt, *L)));
  return FLEP_OK;
}

flep_status flep_debug_copy_events(flep_rt rt, flep_launch_t h, uint32_t epoch,
                                   flep_worker_event* host_out, size_t max_records, size_t* n_out) {
  if (!rt || !host_out) return fail(FLEP_ERR_INVALID, "NULL argument");
  ApiLock lk(rt);
  Launch* L = find(rt, h);
  if (!L) return fail(FLEP_ERR_INVALID, "unknown launch %lld", (long long)h);
  if (!L->dmem) return fail(FLEP_ERR_STATE, "launch resources already released");
  if (epoch == 0 || epoch > L->epoch || L->epoch - epoch >= kEvEpochs)
    return fail(FLEP_ERR_INVALID, "epoch %u not in the log", epoch);
  const size_t n = std::min<size_t>(max_records, L->workers);
  CUDA_TRY(cudaMemcpyAsync(host_out, L->ev + (size_t)((L->gen0 + epoch) % kEvEpochs) * L->workers,
                           n * sizeof(WorkerEvent), cudaMemcpyDeviceToHost, dbg_stream(rt, *L)));
  CUDA_TRY(cudaStreamSynchronize(dbg_stream(rt, *L)));
  // keep only this epoch's records: a slot nobody wrote in this epoch (a CLC CTA that was
  // cancelled, R25) still holds an older generation's record
  const uint32_t gen = L->gen0 + epoch;
  WorkerEvent* r = reinterpret_cast<WorkerEvent*>(host_out);
  size_t m = 0;
  for (size_t i = 0; i < n; ++i)
    if (r[i].epoch == gen) r[m++] = r[i];
  if (n_out) *n_out = m;
  return FLEP_OK;
}

flep_status flep_debug_epoch_info(flep_rt rt, flep_launch_t h, uint32_t epoch, flep_epoch_info* out) {
  if (!rt || !out) return fail(FLEP_ERR_INVALID, "NULL argument");
  ApiLock lk(rt);
  Launch* L = find(rt, h);
  if (!L) return fail(FLEP_ERR_INVALID, "unknown launch %lld", (long long)h);
  if (!L->dmem) return fail(FLEP_ERR_STATE, "launch resources already released");
  if (epoch == 0 || epoch > L->epoch || L->epoch - epoch >= kEvEpochs)
    return fail(FLEP_ERR_INVALID, "epoch %u not in the log", epoch);
  ControlBlock cb;
  CUDA_TRY(cudaMemcpyAsync(&cb, L->cb, sizeof(cb), cudaMemcpyDeviceToHost, dbg_stream(rt, *L)));
  CUDA_TRY(cudaStreamSynchronize(dbg_stream(rt, *L)));
  const uint32_t e = (L->gen0 + epoch) % kEvEpochs;
  out->t_trigger = cb.ep_t_trigger[e];
  // t_end = the epoch's last worker exit. The publishing worker is the last to stop taking work
  // (R23), not necessarily the last to leave, so take the maximum over the epoch's worker log.
  std::vector<WorkerEvent> ev(L->workers);
  CUDA_TRY(cudaMemcpyAsync(ev.data(), L->ev + (size_t)e * L->workers, L->workers * sizeof(WorkerEvent),
                           cudaMemcpyDeviceToHost, dbg_stream(rt, *L)));
  CUDA_TRY(cudaStreamSynchronize(dbg_stream(rt, *L)));
  uint64_t t_end = 0;
  for (const WorkerEvent& w : ev)
    if (w.epoch == L->gen0 + epoch && w.t_exit > t_end) t_end = w.t_exit;
  out->t_end = t_end ? t_end : cb.ep_t_end[e];
  out->trigger_block = cb.ep_trigger_block[e];
  out->done = cb.ep_done[e];
  out->counter = cb.ep_ctr[e];
  out->state = cb.ep_state[e];
  out->relay_smid = L->relay ? cb.ep_relay[e] >> 8 : 0;
  out->relay_reason = L->relay ? cb.ep_relay[e] & 0xffu : 0;
  out->relay_t_exit = L->relay ? cb.ep_relay_t[e] : 0;
  return FLEP_OK;
}

flep_status flep_set_rank_table(flep_rt rt, const uint16_t* rank, uint32_t n) {
  if (!rt || !rank) return fail(FLEP_ERR_INVALID, "NULL argument");
  if (n < rt->nsmid || n > 256) return fail(FLEP_ERR_INVALID, "rank table needs %u entries", rt->nsmid);
  ApiLock lk(rt);
  CUDA_TRY(cudaMemcpyAsync(rt->d_rank, rank, n * sizeof(uint16_t), cudaMemcpyHostToDevice, rt->ctl));
  CUDA_TRY(cudaStreamSynchronize(rt->ctl));
  return FLEP_OK;
}

flep_status flep_decision_log(flep_rt rt, int64_t* out4, size_t max_records, size_t* n_out) {
  if (!rt || !n_out) return fail(FLEP_ERR_INVALID, "NULL argument");
  ApiLock lk(rt);
  if (!rt->policy) { *n_out = 0; return FLEP_OK; }
  const auto& d = rt->policy->decisions();
  const size_t n = std::min(max_records, d.size());
  for (size_t i = 0; i < n && out4; ++i) {
    out4[4 * i] = d[i].t; out4[4 * i + 1] = d[i].action; out4[4 * i + 2] = d[i].id; out4[4 * i + 3] = d[i].n_sms;
  }
  *n_out = out4 ? n : d.size();
  return FLEP_OK;
}

flep_status flep_event_log(flep_rt rt, int64_t* out6, size_t max_records, size_t* n_out) {
  if (!rt || !n_out) return fail(FLEP_ERR_INVALID, "NULL argument");
  ApiLock lk(rt);
  const size_t n = std::min(max_records, rt->evlog.size());
  for (size_t i = 0; i < n && out6; ++i)
    for (int j = 0; j < 6; ++j) out6[6 * i + j] = rt->evlog[i][j];
  *n_out = out6 ? n : rt->evlog.size();
  return FLEP_OK;
}

flep_status flep_event_log_ex(flep_rt rt, int64_t* out7, size_t max_records, size_t* n_out) {
  if (!rt || !n_out) return fail(FLEP_ERR_INVALID, "NULL argument");
  ApiLock lk(rt);
  const size_t n = std::min(max_records, rt->evlog.size());
  for (size_t i = 0; i < n && out7; ++i)
    for (int j = 0; j < 7; ++j) out7[7 * i + j] = rt->evlog[i][j];
  *n_out = out7 ? n : rt->evlog.size();
  return FLEP_OK;
}

// ---- pure policy engine --------------------------------------------------------------------
struct flep_policy_s {
  Policy p;
  flep_policy_s(int32_t k, uint32_t n) : p(k, n) {}
};

flep_status flep_policy_tick(flep_policy_t p, int64_t t, int32_t* acted) {
  if (!p) return fail(FLEP_ERR_INVALID, "NULL policy");
  const bool a = p->p.tick(t);
  if (acted) *acted = a ? 1 : 0;
  return FLEP_OK;
}

flep_status flep_policy_set_max_overhead(flep_policy_t p, uint32_t ppm) {
  if (!p) return fail(FLEP_ERR_INVALID, "NULL policy");
  if (ppm == 0) return fail(FLEP_ERR_INVALID, "max_overhead must be > 0");
  p->p.set_max_overhead_ppm(ppm);
  return FLEP_OK;
}

flep_status flep_policy_create(int32_t kind, uint32_t num_sms, flep_policy_t* out) {
  if (!out) return fail(FLEP_ERR_INVALID, "out is NULL");
  if (kind < kPolicyFIFO || kind > kPolicyREORDER + 1) return fail(FLEP_ERR_INVALID, "bad policy kind %d", kind);
  *out = new flep_policy_s((kind == kPolicySLICE || kind == kPolicyREORDER + 1) ? kPolicyHPF : kind, num_sms);
  return FLEP_OK;
}
flep_status flep_policy_destroy(flep_policy_t p) { delete p; return FLEP_OK; }
flep_status flep_policy_arrive(flep_policy_t p, int64_t t, int64_t id, int32_t prio, int64_t t_e, int64_t o) {
  if (!p) return fail(FLEP_ERR_INVALID, "NULL policy");
  if (p->p.entry(id)) return fail(FLEP_ERR_INVALID, "duplicate id %lld", (long long)id);
  p->p.arrive(t, id, prio, t_e, o);
  return FLEP_OK;
}
flep_status flep_policy_arrive_ex(flep_policy_t p, int64_t t, int64_t id, int32_t prio, int64_t t_e, int64_t o,
                                  int64_t sms_need) {
  if (!p) return fail(FLEP_ERR_INVALID, "NULL policy");
  if (p->p.entry(id)) return fail(FLEP_ERR_INVALID, "duplicate id %lld", (long long)id);
  if (sms_need < 0) return fail(FLEP_ERR_INVALID, "sms_need < 0");
  p->p.arrive(t, id, prio, t_e, o, sms_need);
  return FLEP_OK;
}
flep_status flep_policy_set_spatial(flep_policy_t p, int32_t on) {
  if (!p) return fail(FLEP_ERR_INVALID, "NULL policy");
  p->p.set_spatial(on != 0);
  return FLEP_OK;
}
flep_status flep_policy_finish(flep_policy_t p, int64_t t, int64_t id) {
  if (!p) return fail(FLEP_ERR_INVALID, "NULL policy");
  if (!p->p.entry(id)) return fail(FLEP_ERR_INVALID, "unknown id %lld", (long long)id);
  p->p.finish(t, id);
  return FLEP_OK;
}
flep_status flep_policy_decisions(flep_policy_t p, int64_t* out4, size_t max_records, size_t* n_out) {
  if (!p || !n_out) return fail(FLEP_ERR_INVALID, "NULL argument");
  const auto& d = p->p.decisions();
  const size_t n = std::min(max_records, d.size());
  for (size_t i = 0; i < n && out4; ++i) {
    out4[4 * i] = d[i].t; out4[4 * i + 1] = d[i].action; out4[4 * i + 2] = d[i].id; out4[4 * i + 3] = d[i].n_sms;
  }
  *n_out = out4 ? n : d.size();
  return FLEP_OK;
}

int64_t flep_model_predict_ns(const double m[5], double grid, double cta, double input, double smem) {
  if (!m) return 1;
  const double v = m[0] * grid + m[1] * cta + m[2] * input + m[3] * smem + m[4];
  const double a = v < 0 ? -v : v;
  int64_t r = (int64_t)(a + 0.5);
  if (v < 0) r = -r;
  return r < 1 ? 1 : r;
}

flep_status flep_debug_set_trace(flep_rt rt, void* worker_trace, void* unwrapped_trace) {
  if (!rt) return fail(FLEP_ERR_INVALID, "rt is NULL");
#ifdef FLEP_TRACE
  ApiLock lk(rt);
  rt->trace = (uint64_t*)worker_trace;
  CUDA_TRY(flep::set_unwrapped_trace((uint64_t*)unwrapped_trace));
  return FLEP_OK;
#else
  (void)worker_trace; (void)unwrapped_trace;
  return fail(FLEP_ERR_UNSUPPORTED, "built without FLEP_TRACE");
#endif
}

}  // extern "C"
