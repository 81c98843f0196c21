"""Offline phase of FLEP on B200 (§4.2): per-kernel duration models and preemption
overhead estimates, produced by running the CUDA path and fed to flep_register_kernel.

* Duration model: a per-kernel linear regression with an L2 penalty over four features
  — grid size (original blocks), CTA size, input size (the body's work unit: elements, nonzeros,
  cells, M*N*K) and shared memory per block — trained on randomly sized inputs. Features are
  standardised, the bias is not penalised, lambda = 1 (R14); the fit is returned in raw
  feature units as the 5-vector flep_kernel_desc.model expects.
* Preemption overhead O: the mean, over profiled runs with random preemption points, of
  (preempted-and-resumed duration - uninterrupted duration).

Durations are measured through the same runtime path the policies see (host turnaround of a
standalone launch), L2 flushed before each run.
"""
from __future__ import annotations

import numpy as np

from . import flep as F

DYN_SMEM = {F.BODY_SAXPY_I32: 0, F.BODY_SAXPY_F32: 0, F.BODY_SPMV_CSR_F32: 9 * 1024,
            F.BODY_STENCIL5_F32: 0, F.BODY_STENCIL5_I32: 0, F.BODY_GEMM_BF16: 197 * 1024}


def ridge_fit(X, y, lam: float = 1.0):
    """Ridge regression on standardised features with an unpenalised intercept; returns the
    5-vector [w_grid, w_cta, w_input, w_smem, bias] in raw feature units."""
    X = np.asarray(X, dtype=np.float64)
    y = np.asarray(y, dtype=np.float64)
    mean = X.mean(axis=0)
    scale = X.std(axis=0)
    scale[scale == 0] = 1.0
    Z = (X - mean) / scale
    yc = y - y.mean()
    w = np.linalg.solve(Z.T @ Z + lam * np.eye(Z.shape[1]), Z.T @ yc)
    w_raw = w / scale
    return [float(v) for v in w_raw] + [float(y.mean() - w_raw @ mean)]


def predict(model5, feats):
    f = np.asarray(feats, dtype=np.float64)
    return f @ np.asarray(model5[:4]) + model5[4]


class Workloads:
    """Random-size inputs for each body, carved out of one large allocation per body."""

    def __init__(self, torch, seed=0):
        self.torch = torch
        g = torch.Generator(device="cuda")
        g.manual_seed(seed)
        self.g = g
        self.np_rng = np.random.Generator(np.random.PCG64(seed))
        self.x = torch.rand(1 << 28, device="cuda", generator=g)
        self.y = torch.rand(1 << 28, device="cuda", generator=g)
        R = 1 << 23
        lens = torch.randint(0, 21, (R,), device="cuda", generator=g)
        rowptr = torch.zeros(R + 1, dtype=torch.int64, device="cuda")
        rowptr[1:] = torch.cumsum(lens, 0)
        nnz = int(rowptr[-1])
        rows = torch.repeat_interleave(torch.arange(R, device="cuda"), lens)
        key, _ = torch.sort(rows * R + torch.randint(0, R, (nnz,), device="cuda", generator=g))
        self.col = (key % R).to(torch.int32)
        self.val = torch.rand(nnz, device="cuda", generator=g)
        self.rowptr = rowptr.to(torch.int32)
        self.rowptr_h = rowptr.cpu().numpy()
        self.sy = torch.empty(R, device="cuda")
        self.st_out = torch.empty(16384 * 16384, device="cuda")
        self.ga = (torch.rand(8192 * 8192, device="cuda", generator=g) - 0.5).to(torch.bfloat16)
        self.gb = (torch.rand(8192 * 8192, device="cuda", generator=g) - 0.5).to(torch.bfloat16)
        self.gc = torch.empty(8192 * 8192, device="cuda", dtype=torch.bfloat16)

    def case(self, body, size):
        """(grid, args, feature vector) for one input of the given size."""
        t = self.torch
        if body in (F.BODY_SAXPY_F32,):
            n = int(size)
            grid = F.saxpy_grid(n)
            return grid, F.saxpy_f32_args(self.y[:n], self.x[:n], 0.5), [grid[0], 256, n, DYN_SMEM[body]]
        if body == F.BODY_SPMV_CSR_F32:
            rows = int(size)
            grid = F.spmv_grid(rows)
            nnz = int(self.rowptr_h[rows])
            a = F.SpmvArgs(self.sy.data_ptr(), self.rowptr.data_ptr(), self.col.data_ptr(), self.val.data_ptr(),
                           self.x.data_ptr(), rows)
            return grid, a, [grid[0], 256, nnz, DYN_SMEM[body]]
        if body == F.BODY_STENCIL5_F32:
            n = int(size)
            grid = F.stencil_grid(n)
            a = F.StencilArgs(self.st_out.data_ptr(), self.x.data_ptr(), n)
            return grid, a, [grid[0] * grid[1], 256, n * n, DYN_SMEM[body]]
        if body == F.BODY_GEMM_BF16:
            m = int(size)
            grid = F.gemm_grid(m, m)
            a = F.GemmArgs(self.gc.data_ptr(), self.ga.data_ptr(), self.gb.data_ptr(), m, m, m)
            return grid, a, [grid[0] * grid[1], 256, m * m * m, DYN_SMEM[body]]
        raise ValueError(body)

    def random_size(self, body):
        r = self.np_rng
        if body == F.BODY_SAXPY_F32:
            return int(2 ** r.uniform(16, 28))
        if body == F.BODY_SPMV_CSR_F32:
            return int(2 ** r.uniform(14, 23))
        if body == F.BODY_STENCIL5_F32:
            return int(r.integers(4, 257)) * 64
        if body == F.BODY_GEMM_BF16:
            return int(r.integers(2, 33)) * 256
        raise ValueError(body)


_DITHER = np.random.default_rng(12345)


def dither(torch, base_cycles=0):
    """A spin of random length (0-4096 SM cycles, ~0-2 us) on the current stream before a timed
    launch: CUDA events are stamped with a ~1 us quantum here, and right after the L2 flush the
    launch's phase against that quantum is nearly fixed; the spin randomises it so that the mean
    of the samples resolves well below the quantum (see event_mean_us)."""
    torch.cuda._sleep(int(base_cycles) + int(_DITHER.integers(0, 4096)))


def event_mean_us(ts):
    """Summary of CUDA-event durations (us): events are stamped with a ~1 us quantum on this
    system, so a median of a few samples sits on a quantum; the mean of the middle 80 % of the
    dithered samples (see dither) averages over the quantum instead."""
    v = np.sort(np.asarray(ts, dtype=np.float64))
    k = len(v) // 10
    return float(np.mean(v[k:len(v) - k])) if len(v) > 2 * k else float(np.mean(v))


def _flush(torch, buf):
    buf.zero_()


def measure_duration(rt, kernel, grid, args, torch, flush, reps=2):
    """Median host turnaround (ns) of a standalone launch through the runtime."""
    ts = []
    for _ in range(reps):
        flush()
        torch.cuda.synchronize()
        h = rt.launch(kernel, grid, args)
        rt.sync(h)
        info = rt.query(h)
        ts.append(info.t_finish - info.t_arrive)
    return float(np.median(ts))


def fit_duration_model(rt, torch, wl, body, n_train=100, chunk=1, prefetch=False, flush=None, lam=1.0):
    """Profile `n_train` random inputs (100) and fit the model. Returns (model5, X, y)."""
    k = rt.register_kernel(body, chunk=chunk, poll=1, prefetch=prefetch)
    grid, args, _ = wl.case(body, wl.random_size(body))          # warm-up (first-launch costs)
    for _ in range(3):
        measure_duration(rt, k, grid, args, torch, flush or (lambda: None), reps=1)
    X, y = [], []
    for _ in range(n_train):
        grid, args, feats = wl.case(body, wl.random_size(body))
        X.append(feats)
        y.append(measure_duration(rt, k, grid, args, torch, flush or (lambda: None), reps=1))
    return ridge_fit(X, y, lam), np.array(X, dtype=np.float64), np.array(y)


def preemption_overhead(torch, wl, body, size, runs=50, chunk=1, prefetch=False, flush=None, seed=0):
    """O: mean over `runs` of (preempted-and-resumed - uninterrupted) device span, ns."""
    rt = F.Runtime(exec_on_user_stream=True)
    try:
        k = rt.register_kernel(body, chunk=chunk, poll=1, prefetch=prefetch)
        grid, args, _ = wl.case(body, size)
        nblocks = grid[0] * grid[1]
        rng = np.random.Generator(np.random.PCG64(seed))

        def span(h, epochs):
            evs = []
            for e in range(1, epochs + 1):
                evs += rt.events(h, e)
            return max(e.t_exit for e in evs) - min(e.t_entry for e in evs)

        base = []
        for _ in range(5):
            (flush or (lambda: None))()
            torch.cuda.synchronize()
            h = rt.launch(k, grid, args)
            rt.sync(h)
            base.append(span(h, 1))
        t_alone = float(np.median(base))
        over = []
        for _ in range(runs):
            (flush or (lambda: None))()
            torch.cuda.synchronize()
            rt.arm_next_trigger(int(rng.integers(nblocks // 4, 3 * nblocks // 4)), rt.num_sms)
            h = rt.launch(k, grid, args)
            rt.wait_epoch(h, timeout_ns=10_000_000_000)
            if rt.query(h).state == F.STATE_PREEMPTED:
                rt.resume(h)
                rt.sync(h)
                over.append(span(h, 2) - t_alone)
            else:
                rt.sync(h)
        return int(max(0.0, float(np.mean(over)))) if over else 0, t_alone
    finally:
        rt.close()


# ---- amortizing factor ------------------------------------------------------------------
# "FLEP can automatically find the smallest value for L through offline tuning (trying different
# values from small to large) such that the runtime overhead introduced by the transformation is
# less than 4%." On B200 L = C*K (reading R2): C blocks per counter fetch, a poll every K chunks.
# For one L several variants exist (C vs K split, prefetch, async poll); the tuner tries them from
# the latency-cheapest (no prefetch, synchronous poll) to the throughput-cheapest.

DEFAULT_CANDIDATES = tuple(
    (c, k, pf, ap, clc, sw)
    for c, k in ((1, 1), (2, 1), (1, 2), (4, 1), (2, 2), (1, 4), (8, 1), (4, 2), (16, 1), (8, 2), (32, 1),
                 (16, 2), (64, 1), (32, 4), (200, 1))
    for pf, ap, clc, sw in ((False, False, False, False), (True, False, False, False),
                            (True, True, False, False),
                            (False, False, True, False),     # the CLC task fetch (R25)
                            (False, False, False, True)))    # the scheduling-warp worker (R26)


def select_amortizing_factor(table, bound=0.04):
    """table: iterable of dicts {C, K, prefetch, async_poll, overhead} (overhead as a fraction of
    the unwrapped time). Returns the entry with the smallest L = C*K whose overhead is below
    `bound` (within one L: no prefetch before prefetch, synchronous before async poll — the order
    of added preemption latency — then the lowest overhead), with met=True; if no entry meets the
    bound, the entry with the lowest overhead, met=False."""
    rows = list(table)
    if not rows:
        raise ValueError("empty tuning table")

    def key(r):
        return (r["C"] * r["K"], bool(r["prefetch"]) + bool(r["async_poll"]), r["overhead"])
    # (a CLC variant adds no preemption latency beyond its chunk: it ranks with the plain ones)
    ok = [r for r in rows if r["overhead"] < bound]
    if ok:
        best = min(ok, key=key)
        return dict(best, L=best["C"] * best["K"], met=True)
    best = min(rows, key=lambda r: (r["overhead"], r["C"] * r["K"]))
    return dict(best, L=best["C"] * best["K"], met=False)


def tune_amortizing_factor(rt, torch, body, grid, args, flush, bound=0.04, candidates=DEFAULT_CANDIDATES,
                           reps=30, stream=None):
    """Offline tuning of L for one kernel and input: time the unwrapped kernel and the
    wrapped variants (CUDA events on `stream`, L2 flushed before each launch, trimmed mean of `reps`),
    trying L from small to large and stopping at the first L that has a variant under `bound`.
    `rt` must be a MANUAL-mode runtime with exec_on_user_stream. Returns (choice, table)."""
    s = stream or torch.cuda.current_stream()

    def timed(fn):
        ts = []
        for r in range(reps + 2):
            with torch.cuda.stream(s):
                flush()
                dither(torch)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            h = fn()
            e1.record(s)
            e1.synchronize()
            if h is not None:
                rt.sync(h)
            if r >= 2:
                ts.append(e0.elapsed_time(e1) * 1e3)
        return event_mean_us(ts)

    t_u = timed(lambda: rt.launch_unwrapped(body, grid, args, stream=s))
    table = []
    by_l = {}
    for cand in candidates:
        c, k, pf, ap, clc, sw = (tuple(cand) + (False, False))[:6]
        if body == F.BODY_GEMM_BF16 and (pf or clc or sw):
            continue                          # in-tile GEMM: no prefetch, CLC or scheduling warp
        if body == F.BODY_STENCIL5_F32_TMA and sw:
            continue                          # the TMA stencil synchronises the whole CTA in run()
        by_l.setdefault(c * k, []).append((c, k, pf, ap, clc, sw))
    for L in sorted(by_l):
        for c, k, pf, ap, clc, sw in by_l[L]:
            kk = rt.register_kernel(body, chunk=c, poll=k, prefetch=pf, async_poll=ap,
                                    in_tile=body == F.BODY_GEMM_BF16, clc=clc, sched_warp=sw)
            t_w = timed(lambda: rt.launch(kk, grid, args, stream=s))
            table.append({"C": c, "K": k, "prefetch": pf, "async_poll": ap, "clc": clc, "sched_warp": sw,
                          "wrapped_us": round(t_w, 3), "unwrapped_us": round(t_u, 3),
                          "overhead": t_w / t_u - 1.0})
        if any(r["overhead"] < bound for r in table if r["C"] * r["K"] == L):
            break
    return select_amortizing_factor(table, bound), table
