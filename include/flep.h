/*
 * flep.h — C ABI of the B200-native FLEP runtime (preemptable persistent-CTA kernels).
 *
 * Paper: Wu, Liu, Zhou, Jiang, "FLEP: Enabling Flexible and Efficient Preemption on GPUs",
 * ASPLOS'17. "P:N" = line N of the paper text.
 *
 * What the library does: a registered kernel is launched as a grid of
 * resident worker CTAs (persistent threads) that pull chunks of C original
 * block indices from a global atomic counter (pull_task, Fig. 4), run the
 * original block body on each, and poll a 32-bit control word every K chunks (amortized check,
 * Fig. 4(b)). On a preemption request either all workers exit (temporal, Fig. 4(a/b),
 * P:164) or only those whose SM is among the n released ones (spatial, Fig. 4(c)).
 * Progress lives in the counter, so a resume launch runs every original block exactly once
 * (P:126). A host runtime intercepts launches and, in managed modes,
 * decides who is preempted and when (HPF/SRPT, Fig. 6, §5.2; FIFO and kernel-slicing baselines).
 *
 * Conventions (all functions):
 *   - Return flep_status: 0 = FLEP_OK, < 0 = error. Never throw, never abort. After an error,
 *     flep_last_error() returns a thread-local human-readable message.
 *   - A sticky CUDA error makes every later call return FLEP_ERR_CUDA; re-initialise.
 *   - Device pointers passed inside argument structs belong to the caller and must stay valid
 *     until flep_sync() has returned FLEP_OK for that launch. Argument structs are copied by
 *     value at flep_launch().
 *   - The runtime owns its control blocks, internal CUDA streams (one high-priority control
 *     stream, a pool of execution streams) and pinned host status words.
 *   - flep_launch / flep_preempt / flep_resume are asynchronous. Work the caller enqueued on
 *     `stream` BEFORE flep_launch precedes the workers (event dependency). Completion (every
 *     block done, possibly after several preempt/resume cycles) is observable through
 *     flep_sync / flep_query; the runtime never blocks a stream on a device-written value
 *     (front-end waits can deadlock when streams share a hardware queue).
 *   - Priority: larger value = higher priority (Fig. 6 line 1: Kr.priority < Kn.priority ->
 *     preempt). The runtime maps it onto CUDA stream priorities internally.
 *   - One runtime per device; all entry points are thread-safe (internal mutex).
 */
#ifndef FLEP_H
#define FLEP_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  FLEP_OK = 0,
  FLEP_ERR_INVALID = -1,      /* bad argument: n_sms == 0, empty grid, unknown body/kernel/handle */
  FLEP_ERR_STATE = -2,        /* operation not allowed in the launch's current state / mode */
  FLEP_ERR_CUDA = -3,         /* CUDA runtime/driver error (message in flep_last_error) */
  FLEP_ERR_NOMEM = -4,        /* device or pinned host allocation failed */
  FLEP_ERR_TIMEOUT = -5,      /* flep_sync timeout expired (launch still in flight) */
  FLEP_ERR_UNSUPPORTED = -6   /* feature not available on this device/build */
} flep_status;

typedef struct flep_rt_s* flep_rt;   /* one runtime per GPU */
typedef int32_t flep_kernel;          /* registered kernel id (>= 0) */
typedef int64_t flep_launch_t;        /* one invocation (>= 1); handle for preempt/resume/sync */
typedef void* flep_stream_t;          /* a cudaStream_t (NULL = legacy default stream) */

typedef struct { uint32_t x, y, z; } flep_dim3;

typedef enum {
  FLEP_POLICY_MANUAL = 0,  /* caller issues preempt/resume itself (mechanism only) */
  FLEP_POLICY_FIFO = 1,    /* interception, no preemption, arrival order (MPS co-run baseline) */
  FLEP_POLICY_HPF = 2,     /* Fig. 6: priority preemption + SRPT within a priority (§5.2.1) */
  FLEP_POLICY_SLICE = 3,   /* HPF decisions on the kernel-slicing mechanism (P:96, P:391 baseline) */
  FLEP_POLICY_FFS = 4,     /* fairness first under an overhead constraint: weighted round robin,
                              epoch T*W_i, W_i = priority+1, T minimal with
                              sum O_i / (T sum W_i) <= max_overhead (§5.2.2) */
  FLEP_POLICY_REORDER = 5, /* kernel-reordering baseline without preemption: shortest queued kernel
                              of the highest priority runs next */
  FLEP_POLICY_SLICE_DEVICE = 6 /* HPF decisions on kernel slicing with every slice enqueued at
                              launch and a device-side check at slice entry (the first CTA of a
                              slice decides for all of it: run, or skip when a request is in
                              force), so a never-preempted kernel pays only the launch gaps
                              between its slices (R31; P:96, P:391 baseline) */
} flep_policy;

typedef enum {
  FLEP_FLAG_STREAM_MEMOP = 0,  /* ctrl word in device memory, written by cuStreamWriteValue32 on a
                                  high-priority control stream (needs no SM) */
  FLEP_FLAG_HOST_MAPPED = 1    /* ctrl word in mapped pinned host memory, written by a CPU store
                                  (the paper's temp_P in pinned memory) */
} flep_flag_transport;

typedef enum {
  FLEP_BODY_SAXPY_I32 = 1,     /* y <- a*x + y, int32, wraps mod 2^32; 256 elements per block */
  FLEP_BODY_SAXPY_F32 = 2,     /* y <- a*x + y, fp32; 256 elements per block */
  FLEP_BODY_SPMV_CSR_F32 = 3,  /* y = A x, CSR fp32; 128 rows per block */
  FLEP_BODY_STENCIL5_F32 = 4,  /* 5-point out-of-place sweep, fp32; 64x64 cells per block */
  FLEP_BODY_STENCIL5_I32 = 5,  /* 5-point integer sweep, wraps mod 2^32; 64x64 cells per block */
  FLEP_BODY_GEMM_BF16 = 6,     /* C = A B^T, bf16 in, fp32 accumulate (tcgen05), bf16 out;
                                  128x256 output tile per block */
  FLEP_BODY_STENCIL5_F32_TMA = 7, /* STENCIL5_F32 with the tile and its halo staged in shared memory
                                  by the TMA unit and the output tile written back by a bulk
                                  tensor store; same args; n % 4 == 0, 16-byte aligned in/out */
  FLEP_BODY_SPMV_CSR_F32_VEC = 8, /* y = A x, CSR fp32, CSR-vector form (4 lanes per row, shuffle
                                  reduction, no shared memory); same args; 128 rows per block,
                                  each warp owns 16 of them (warp-task capable, R30) */
  FLEP_BODY_GEMM_BF16_2SM = 9, /* GEMM_BF16 on CTA pairs (cluster of 2, tcgen05.mma.cta_group::2):
                                  256x256 output tile per block, grid (N/256, M/256, 1),
                                  M % 256 == N % 256 == K % 64 == 0; the worker is the pair
                                  (flep_launch_info.workers = pairs), tile-granular preemption, a
                                  spatial request releases a pair iff it names either SM (R32) */
  FLEP_BODY_GEMM_BF16_2SM_W = 10 /* GEMM_BF16_2SM with a 256x512 output tile per block (two
                                  N = 256 MMAs per k-slice into one 512-column TMEM accumulator):
                                  grid (N/512, M/256, 1), M % 256 == N % 512 == K % 64 == 0;
                                  a quarter less L2 -> SM operand traffic per flop than the
                                  256x256 tile, no overlap of one tile's epilogue with the next
                                  tile's MMAs; in-tile preemption spills 256 KiB per CTA */
} flep_body;

/* Per-body argument structs (copied by value at launch). All pointers are device pointers. */
typedef struct { int32_t* y; const int32_t* x; int32_t a; uint32_t n; } flep_saxpy_i32_args;
typedef struct { float* y; const float* x; float a; uint32_t n; } flep_saxpy_f32_args;
typedef struct {
  float* y; const int32_t* rowptr; const int32_t* col; const float* val; const float* x;
  uint32_t rows;
} flep_spmv_args;
/* in/out: n x n row-major, float (STENCIL5_F32) or int32 (STENCIL5_I32); out != in. */
typedef struct { void* out; const void* in; uint32_t n; } flep_stencil_args;
/* a: M x K row-major bf16, b: N x K row-major bf16 (K-major "TN"), c: M x N row-major bf16.
   M % 128 == 0, N % 256 == 0, K % 64 == 0. */
typedef struct { void* c; const void* a; const void* b; uint32_t m, n, k; } flep_gemm_args;

typedef struct {
  int32_t policy;              /* flep_policy */
  int32_t flag;                /* flep_flag_transport */
  uint32_t default_chunk;      /* C: original blocks per counter fetch (0 -> 8) */
  uint32_t default_poll;       /* K: chunks between control-word polls (0 -> 1) */
  uint32_t debug_coverage;     /* bit 0: keep a per-block execution count cov[N] (test builds);
                                  any non-zero value: keep the device logs (worker events, epoch
                                  summaries) of the newest 64 finished launches for the debug
                                  copies (2 = logs only, no coverage count in the workers) */
  uint32_t spatial;            /* HPF only: 1 = the runtime decides how far to preempt: a
                                  higher-priority arrival that needs n < num_sms SMs
                                  (n = ceil(workers / resident CTAs per SM), A9)
                                  gets a spatial yield of n SMs and runs beside the victim, which
                                  is refilled to every SM when it finishes (R29);
                                  0 = always temporal (Fig. 6 as printed) */
  uint32_t slice_blocks;       /* SLICE policy: blocks per sub-kernel (0 -> W*C*K, A20) */
  uint32_t exec_on_user_stream;/* launch worker grids (and resumes, slices) directly on the
                                  caller's stream instead of a runtime stream. Stream order then
                                  only covers the epoch grids: the caller must resume (manual) or
                                  sync (managed) before enqueuing work that depends on the
                                  results. In managed modes this is a measurement aid (CUDA events
                                  on the caller's stream bracket a launch the policy starts at
                                  once). */
  uint32_t max_overhead_ppm;   /* FFS: max_overhead in parts per million (0 -> 100000 = 10%) */
} flep_options;

typedef struct {
  const char* name;
  int32_t body;                /* flep_body */
  uint32_t chunk, poll;        /* C, K (0 = runtime defaults) */
  double model[5];             /* ridge model: T_e ns = m0*grid + m1*cta + m2*input
                                  + m3*smem + m4, rounded once to integer ns */
  int64_t preempt_overhead_ns; /* O: profiled mean preemption overhead */
  uint32_t flags;              /* FLEP_KFLAG_* */
  uint32_t ctas_per_sm;        /* resident workers per SM (0 = the occupancy maximum) */
} flep_kernel_desc;

/* Prefetch the next chunk's index while the current chunk runs (hides the counter atomic's
   latency; a worker that must yield still executes the chunk it holds, so the drain can take up
   to one extra chunk). */
#define FLEP_KFLAG_PREFETCH 1u
/* The first worker of every epoch publishes "epoch started" to the launch's pinned status slot
   (flep_launch_info.started_epoch). Off by default: the system-scope store it needs delays the
   grid's completion by about a microsecond. */
#define FLEP_KFLAG_STARTED_HINT 2u
/* In-tile preemption (GEMM bodies only; not with FLEP_KFLAG_PREFETCH): workers also poll inside a
   tile (every 4 k-steps) and, when asked to leave, spill the fp32 accumulator of the tile in
   progress to a per-worker slot; the next epoch's worker with the same index restores it and
   continues the k-loop. The result stays bit-identical to an uninterrupted run. Costs
   W x (16 B + 128 KiB) of device memory per launch (runtime-owned, pooled); for the CTA-pair
   body (FLEP_BODY_GEMM_BF16_2SM) one record per pair and one 128 KiB slot per CTA (each CTA
   spills its 128-row half of the 256x256 tile); for the wide pair body
   (FLEP_BODY_GEMM_BF16_2SM_W) two 128 KiB slots per CTA (its 128x512 half).
   flep_register_kernel returns FLEP_ERR_UNSUPPORTED for other bodies or with prefetch. */
#define FLEP_KFLAG_IN_TILE 4u
/* Asynchronous poll: the control word a worker tests at a poll point was loaded at its previous
   scheduling step, so no L2 round trip sits between two chunks; a request is acted on up to one
   chunk later. For throughput-oriented kernels (with FLEP_KFLAG_PREFETCH the scheduling step then
   waits on nothing). */
#define FLEP_KFLAG_ASYNC_POLL 8u
/* CLC task fetch (R25; memory-bound bodies only, not GEMM): the launch runs
   the original grid in chunks (ceil(N/C) CTAs, CTA i = original blocks [iC, iC+C)); a running CTA
   runs its own chunk and then takes pending CTAs' chunks by cancelling them with the hardware's cluster launch control (try_cancel) instead of
   an atomic counter. flep_preempt makes the named workers stop taking blocks at their next poll
   (every K blocks) and leave; the rest of the grid waits in the hardware queue, where
   higher-priority streams are served first. The launch goes to PREEMPTED (temporal) or PARTIAL
   (spatial) at once; flep_resume withdraws the request (no relaunch); completion is the grid's
   completion. The worker event log covers the first W CTAs. */
#define FLEP_KFLAG_CLC 16u
/* Scheduling-warp worker (R26; bodies without whole-CTA barriers in run(): SAXPY, SpMV,
   register stencils): the poll/fetch/exit step runs in one extra warp that keeps the next chunk in
   a shared-memory ring, one chunk ahead (as FLEP_KFLAG_PREFETCH), so the body warps never wait
   for it. The CTA is kThreads + 32 threads (fewer resident CTAs per SM may fit). */
#define FLEP_KFLAG_SCHED_WARP 32u
/* Request relay (R28; plain counter worker of the memory-bound bodies, stream-memop
   transport): the grid gets one extra CTA that is not a worker; its thread polls the launch's
   pinned slot, where every request is also stored, and copies each new value into the device
   control word, so a request reaches the workers in ~1 us instead of waiting for the stream memop
   (~5 us, tens of us behind copy-engine work). Takes one resident slot (W = k x SMs - 1). */
#define FLEP_KFLAG_HOST_RELAY 64u
/* Warp-task worker (R30; STENCIL5_F32/I32 and SPMV_CSR_F32_VEC, not with CLC,
   scheduling warp, in-tile or the SLICE policy): the unit of work is one warp's share of an
   original block (task = block x 8 + warp) and every warp of a worker CTA fetches, polls and
   exits on its own, so no warp waits for another at a chunk boundary and a request is acted on
   after one warp task. For these launches the counter, the coverage log, the done count
   (flep_launch_info.blocks_total / blocks_done / counter), the chunk C and the debug trigger's
   block index are in tasks (flep_launch_info.tasks_per_block = 8; the trigger index given in
   blocks is converted); worker records are per warp. */
#define FLEP_KFLAG_WARP_TASKS 128u
/* In-chunk stop (R33; the counter worker of the memory-bound bodies, not with prefetch,
   CLC, the scheduling warp, warp tasks or in-tile): chunks of C blocks per fetch, and a poll
   between the blocks of a chunk (async, R22), so a request is acted on after one block whatever
   C is. A worker stopped mid-chunk leaves the rest of its chunk in a per-worker record that the
   worker with the same index runs first in the next epoch (a preempted epoch's coverage is then
   not a prefix of the counter). Costs W x 16 B of runtime-owned device memory. */
#define FLEP_KFLAG_IN_CHUNK 256u
/* Speculative fetch (counter worker of the memory-bound bodies, R34): at a poll point
   the worker issues the task-fetch atomic and the poll load together (one L2 round trip on the
   scheduling step instead of two back to back). A worker that must leave after fetching returns
   the unstarted chunk through its per-worker record (as FLEP_KFLAG_IN_CHUNK), which the worker
   with the same index runs first in the next epoch: a request still costs at most one chunk.
   Not with FLEP_KFLAG_PREFETCH, FLEP_KFLAG_ASYNC_POLL, FLEP_KFLAG_CLC, FLEP_KFLAG_SCHED_WARP,
   FLEP_KFLAG_WARP_TASKS or FLEP_KFLAG_IN_TILE (FLEP_KFLAG_IN_CHUNK workers always fetch this way);
   flep_register_kernel returns FLEP_ERR_UNSUPPORTED otherwise. Costs W x 16 B of runtime-owned
   device memory; a preempted epoch's coverage is then not a prefix of the counter. */
#define FLEP_KFLAG_SPEC_FETCH 512u

typedef enum {
  FLEP_STATE_QUEUED = 0,     /* intercepted, waiting for a scheduling decision (S2) */
  FLEP_STATE_RUNNING = 1,    /* workers launched, no request pending (S3) */
  FLEP_STATE_YIELDING = 2,   /* temporal request issued, epoch not yet drained */
  FLEP_STATE_PREEMPTED = 3,  /* epoch drained with blocks left; resumable */
  FLEP_STATE_PARTIAL = 4,    /* spatial request in force: running on the non-released SMs */
  FLEP_STATE_DONE = 5        /* every original block executed exactly once */
} flep_state;

typedef struct {
  int32_t state;               /* flep_state */
  uint32_t epoch;              /* number of worker grids launched so far (1 after first launch) */
  uint64_t blocks_total;       /* N */
  uint64_t blocks_done;        /* done counter as of the last drained epoch */
  uint64_t counter;            /* task counter value (may exceed N by <= W*C, A5) */
  int64_t t_e, t_w, t_r;       /* execution-status triplet, ns (§5.1) */
  int64_t t_arrive, t_first_start, t_finish;  /* host steady clock, ns */
  uint32_t workers;            /* W: worker CTAs per epoch */
  uint32_t n_yield;            /* yield width currently requested (0 = none) */
  int64_t t_last_request;      /* host ns of the last preempt request issued by the runtime */
  int64_t t_last_drain;        /* host ns the runtime observed the last PREEMPTED epoch end */
  uint32_t started_epoch;      /* newest epoch (1-based) whose first worker has begun running
                                  (kernels registered with FLEP_KFLAG_STARTED_HINT; else 0) */
  uint32_t tasks_per_block;    /* 1, or 8 for FLEP_KFLAG_WARP_TASKS launches (counts are in tasks) */
} flep_launch_info;

/* Per-worker event record of one epoch (device %globaltimer, ns). */
typedef struct {
  uint32_t smid;      /* %smid the worker ran on */
  uint32_t reason;    /* 1 = yielded on request, 2 = counter exhausted */
  uint32_t n_blocks;  /* original blocks this worker executed */
  uint32_t epoch;     /* epoch the record belongs to */
  uint64_t t_entry;   /* worker start */
  uint64_t t_exit;    /* worker exit */
} flep_worker_event;

/* Per-epoch device summary. */
typedef struct {
  uint64_t t_trigger;      /* device self-trigger time (0 if none fired this epoch) */
  uint64_t t_end;          /* last worker exit of the epoch */
  uint32_t trigger_block;  /* block index that fired it */
  uint32_t done;           /* done counter at epoch end */
  uint32_t counter;        /* task counter at epoch end */
  uint32_t state;          /* 3 = PREEMPTED, 5 = DONE */
  uint32_t relay_smid;     /* FLEP_KFLAG_HOST_RELAY: SM of the epoch's relay CTA */
  uint32_t relay_reason;   /* why it left: 1 = a spatial request released its SM, 2 = it relayed
                              a temporal request, 3 = the epoch was published; 0 = no relay */
  uint64_t relay_t_exit;   /* when it left (%globaltimer) */
} flep_epoch_info;

/* ---- lifecycle ------------------------------------------------------------------------ */
/* Create the runtime for CUDA device `device`. opts may be NULL (defaults). */
flep_status flep_init(int device, const flep_options* opts, flep_rt* out);
/* Cancel every unfinished launch (unblocking waiting streams), synchronise, free everything. */
flep_status flep_shutdown(flep_rt rt);
/* num_sms = multiprocessor count; nsmid = %nsmid upper bound of %smid values. */
flep_status flep_device_info(flep_rt rt, uint32_t* num_sms, uint32_t* nsmid);

/* ---- user-defined bodies (extension; the paper transforms any kernel) ------------
   A body written in the caller's own .cu against include/flep_body.cuh (a struct with Args,
   kThreads, kMinBlocks and `run(args, b0, b1, gx, gy)` running original blocks [b0, b1), plus
   setup/teardown) gets the FLEP worker, the original (unwrapped) grid and the static twin
   instantiated there by FLEP_DEFINE_BODY(sym, Body), which also defines `sym_ops(flep_body_ops*)`.
   flep_register_body copies the table and returns a body id (>= FLEP_BODY_USER_FIRST) usable in
   flep_kernel_desc.body like a built-in one: counter worker (chunk C, poll K), temporal and
   spatial preemption, resume, managed policies, the CLC fetch and slicing with the device
   check. Not available to user bodies: the scheduling-warp / warp-task / in-chunk workers and
   in-tile preemption. The caller's .cu must be compiled against the same flep headers as libflep.so
   (abi_version), for sm_100a, and its module must stay loaded while the runtime uses the body.
   Errors: FLEP_ERR_INVALID for NULL or incomplete tables, a zero or > 1024 thread count, a
   mismatched abi_version; FLEP_ERR_NOMEM when FLEP_BODY_USER_MAX bodies are registered. */
#define FLEP_BODY_USER_FIRST 64
#define FLEP_BODY_USER_MAX 16
#define FLEP_BODY_ABI_VERSION 1u
typedef struct {
  uint32_t abi_version;        /* FLEP_BODY_ABI_VERSION */
  uint32_t threads;            /* CTA size of the body (Body::kThreads) */
  size_t args_size;            /* sizeof(Body::Args): flep_launch's args_size must match */
  const char* name;
  /* cudaError_t-valued launchers (0 = success) generated by FLEP_DEFINE_BODY: W worker CTAs with
     the runtime's (opaque) worker parameters; the original grid or its 1-D slice
     [offset, offset + count); the static persistent twin; resident worker CTAs per SM */
  int (*worker)(const void* args, const void* worker_params, uint32_t ctas, flep_stream_t stream, int coverage);
  int (*unwrapped)(const void* args, flep_dim3 grid, uint32_t offset, uint32_t count, flep_stream_t stream);
  int (*static_launch)(const void* args, flep_dim3 grid, uint32_t ctas, uint32_t chunk, flep_stream_t stream);
  int (*occupancy)(int* ctas_per_sm, int coverage);
  /* optional (NULL = unsupported): the CLC worker over the original grid in chunks
     (FLEP_KFLAG_CLC), and the device-checked slice kernel (FLEP_POLICY_SLICE_DEVICE) with the
     runtime's (opaque) slice parameters */
  int (*clc)(const void* args, const void* worker_params, uint32_t ctas, flep_stream_t stream, int coverage);
  int (*sliced)(const void* args, flep_dim3 grid, uint32_t offset, uint32_t count, const void* slice_params,
                flep_stream_t stream);
} flep_body_ops;
flep_status flep_register_body(flep_rt rt, const flep_body_ops* ops, int32_t* body_out);

/* ---- kernels and launches ------------------------------------------------------------- */
flep_status flep_register_kernel(flep_rt rt, const flep_kernel_desc* desc, flep_kernel* out);
/* Intercepted launch: `grid` is the ORIGINAL grid in blocks; `args` points to the
   body's argument struct of exactly `args_size` bytes. In MANUAL mode the workers are launched
   immediately; in managed modes the policy decides (launch now, preempt the running kernel,
   or queue). */
flep_status flep_launch(flep_rt rt, flep_kernel k, flep_dim3 grid, const void* args,
                        size_t args_size, int32_t priority, flep_stream_t stream,
                        flep_launch_t* out);
/* MANUAL mode only. Ask a running launch to yield n_sms SMs (n_sms >= num_sms: temporal,
   P:174). Within one epoch a request can only widen. FLEP_ERR_INVALID if n_sms == 0. */
flep_status flep_preempt(flep_rt rt, flep_launch_t h, uint32_t n_sms);
/* MANUAL mode only. PREEMPTED: relaunch the workers on the same counter (stream-ordered after
   the drained grid). PARTIAL: withdraw the spatial request (the remaining workers continue). */
flep_status flep_resume(flep_rt rt, flep_launch_t h);
/* MANUAL mode only. Spatial refill: for a PARTIAL launch, widen the request to the
   whole GPU for the running epoch and queue a full-width epoch behind it, so the victim is
   re-spread over every SM once the waiting kernel is done (the paper's baseline keeps it on the
   remaining SMs). If the running epoch completes the launch first, the refill epoch
   exits without work. PREEMPTED: same as flep_resume. */
flep_status flep_refill(flep_rt rt, flep_launch_t h);
/* Wait until the launch is DONE (timeout_ns < 0: forever). Also waits for its last grid. */
flep_status flep_sync(flep_rt rt, flep_launch_t h, int64_t timeout_ns);
/* Refresh and return the launch's state (never blocks). */
flep_status flep_query(flep_rt rt, flep_launch_t h, flep_launch_info* out);
/* Abandon a launch: temporal preempt, drain, mark done so no stream waits forever. */
flep_status flep_cancel(flep_rt rt, flep_launch_t h);
/* Wait for the current epoch of h to drain (state leaves RUNNING/YIELDING/PARTIAL). */
flep_status flep_wait_epoch(flep_rt rt, flep_launch_t h, int64_t timeout_ns);

/* ---- baselines (same bodies, no wrapper) ----------------------------------------------- */
/* The original kernel: one CTA per original block (unwrapped twin, K7). */
flep_status flep_launch_unwrapped(flep_rt rt, int32_t body, flep_dim3 grid, const void* args,
                                  size_t args_size, flep_stream_t stream);
/* Kernel slicing (K8): ceil(N/slice_blocks) back-to-back sub-kernels of slice_blocks. */
flep_status flep_launch_sliced(flep_rt rt, int32_t body, flep_dim3 grid, const void* args,
                               size_t args_size, uint32_t slice_blocks, flep_stream_t stream);
/* The static persistent twin (U1): the body's resident CTAs (pairs for GEMM_BF16_2SM) take chunks
   of `chunk` blocks in a fixed round-robin order, with no counter, no poll, no exit accounting:
   persistence without the FLEP wrapper, the baseline that isolates the wrapper's own cost.
   FLEP_ERR_UNSUPPORTED for bodies without it (the TMA stencil). */
flep_status flep_launch_static(flep_rt rt, int32_t body, flep_dim3 grid, const void* args,
                               size_t args_size, uint32_t chunk, flep_stream_t stream);
/* Worker grid size W (= resident CTAs per SM x SMs) for a body / chunk. */
flep_status flep_workers_for(flep_rt rt, int32_t body, uint32_t* ctas_per_sm, uint32_t* workers);

/* ---- test / bench hooks (always compiled; cost nothing when unused) -------------------- */
/* Device self-trigger: the worker that fetches the chunk holding `block_index` writes the
   request (epoch, n_sms) itself and stamps the time (flep_epoch_info.t_trigger). n_sms == 0 only
   stamps the time (an arrival marker, no request). Applies to the launch's next epoch if it is
   not running. */
flep_status flep_debug_trigger_at(flep_rt rt, flep_launch_t h, uint64_t block_index,
                                  uint32_t n_sms);
/* Arm a self-trigger for the NEXT flep_launch issued on this runtime. */
flep_status flep_debug_arm_next_trigger(flep_rt rt, uint64_t block_index, uint32_t n_sms);
/* Copy cov[0..n) (debug_coverage runtimes only). */
flep_status flep_debug_copy_coverage(flep_rt rt, flep_launch_t h, uint32_t* host_out, size_t n);
/* Copy the worker event records of epoch `epoch` (1-based; the last 8 epochs are kept): up to
   max_records records written in that epoch, compacted to the front of host_out; *n_out = their
   number (a CLC launch logs the first W CTAs of its grid that ran, R25). */
flep_status flep_debug_copy_events(flep_rt rt, flep_launch_t h, uint32_t epoch,
                                   flep_worker_event* host_out, size_t max_records,
                                   size_t* n_out);
flep_status flep_debug_epoch_info(flep_rt rt, flep_launch_t h, uint32_t epoch,
                                  flep_epoch_info* out);
/* Diagnostics builds (-DFLEP_TRACE) only, else FLEP_ERR_UNSUPPORTED: record per-chunk scheduling
   timestamps of worker grids (device buffer [W][64][5] u64: tid 0 reaches the scheduling step,
   the poll decision, the step returns, the chunk barrier releases, the chunk base is known) and
   entry/exit of every block of unwrapped grids ([N][2] u64). Buffers are
   the caller's; NULL disables. */
flep_status flep_debug_set_trace(flep_rt rt, void* worker_trace, void* unwrapped_trace);
/* Set the spatial rank table: rank[smid] for smid < nsmid (default rank = smid). */
flep_status flep_set_rank_table(flep_rt rt, const uint16_t* rank, uint32_t n);
/* Host steady-clock now, ns (the clock all host timestamps use). */
int64_t flep_now_ns(void);
/* Decision log of the managed runtime: n records of (t_ns, action, launch, n_sms) with
   action 0 = LAUNCH, 1 = RESUME, 2 = PREEMPT (n_sms = yield width: num_sms temporal, fewer
   spatial), 3 = REFILL (a spatially preempted launch back on every SM); and the event log
   (t_ns, type, launch) with type 0 = ARRIVE, 1 = FINISH, 2 = TICK (FFS epoch expiry;
   launch = -1), plus per-launch (priority, t_e, overhead). out4 / out6 may be NULL: *n_out is
   then the number of records available. */
flep_status flep_decision_log(flep_rt rt, int64_t* out4, size_t max_records, size_t* n_out);
flep_status flep_event_log(flep_rt rt, int64_t* out6, size_t max_records, size_t* n_out);
/* The event log with a 7th field per record: the SMs the launch needs (ARRIVE records; the
   spatial HPF input, A9), else 0. */
flep_status flep_event_log_ex(flep_rt rt, int64_t* out7, size_t max_records, size_t* n_out);

/* ---- pure policy engine (host only; no GPU needed) -------------------------------------
   The exact decision logic the managed runtime uses (Fig. 6), exposed for replay parity with
   the oracle's discrete-event simulation. kind: 1 FIFO, 2 HPF, 3 SLICE (= HPF decisions), 4 FFS,
   5 REORDER, 6 SLICE_DEVICE (= HPF decisions). */
typedef struct flep_policy_s* flep_policy_t;
flep_status flep_policy_create(int32_t kind, uint32_t num_sms, flep_policy_t* out);
flep_status flep_policy_destroy(flep_policy_t p);
flep_status flep_policy_arrive(flep_policy_t p, int64_t t_ns, int64_t id, int32_t priority,
                               int64_t t_e_ns, int64_t overhead_ns);
/* Same, with the SMs the kernel needs (spatial HPF input; 0 = the whole GPU). */
flep_status flep_policy_arrive_ex(flep_policy_t p, int64_t t_ns, int64_t id, int32_t priority,
                                  int64_t t_e_ns, int64_t overhead_ns, int64_t sms_need);
/* HPF (kind 2): 1 = spatial preemption decisions (R29), 0 = temporal only (default). */
flep_status flep_policy_set_spatial(flep_policy_t p, int32_t on);
flep_status flep_policy_finish(flep_policy_t p, int64_t t_ns, int64_t id);
/* Decisions emitted so far: records of 4 int64 (t_ns, action, id, n_sms); action as in
   flep_decision_log. */
flep_status flep_policy_decisions(flep_policy_t p, int64_t* out4, size_t max_records,
                                  size_t* n_out);
/* FFS (kind 4): epoch-expiry check at time t; *acted = 1 iff it changed the schedule.
   Other kinds: no-op. */
flep_status flep_policy_tick(flep_policy_t p, int64_t t_ns, int32_t* acted);
/* FFS max_overhead in ppm (default 100000). */
flep_status flep_policy_set_max_overhead(flep_policy_t p, uint32_t ppm);
/* T_e ns from a 5-term model, rounded once (half away from zero), clamped >= 1. */
int64_t flep_model_predict_ns(const double model[5], double grid, double cta, double input,
                              double smem);

const char* flep_last_error(void);
const char* flep_version(void);

#ifdef __cplusplus
}
#endif
#endif /* FLEP_H */
