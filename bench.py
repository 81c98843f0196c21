#!/usr/bin/env python
"""FLEP-on-B200 benchmark (driver contract: one JSON line from rank 0).

Default workload = BASELINE.json configs[1]: a long low-priority fp32 SpMV-CSR (2^20 rows,
~10.5M nnz) is temporally preempted mid-run (full-GPU yield) by a short high-priority 5-point
fp32 stencil (4096^2), then resumed. One STEP = one whole co-run: LP launch -> preemption
request at a seeded block t* (device self-trigger, uniform over the middle half) -> LP drains ->
HP (which arrives with the request) runs -> LP resumes and finishes. Every §8(a) step runs
inside the timed region: launch sizing, worker entry, chunk fetch, body, poll, progress record,
yield, resume.

Headline `value` (metric = BASELINE.json's): the full-GPU preemption latency in us, measured on
the device (%globaltimer): request visible on the GPU -> last victim CTA gone, i.e. all 148 SMs
released (median over the timed steps; max over ranks). Also reported: the waiting kernel's
start latency (request -> its first CTA running), wrapper overhead (wrapped vs unwrapped kernel time), the roofline of the
dominant kernel, the oracle on the host cores, and an end-to-end number through the managed
(HPF) public API with host buffers.

Other configs: --config corun1 | spatial | queue.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from synth import gen  # noqa: E402
from paper_conf_asplos_wulzj17_b200.calibrate import dither, event_mean_us  # noqa: E402

METRIC = ("preemption latency µs (full vs N-SM yield); wrapper overhead % of HBM/tensor roofline; "
          "co-run NATT")
HBM_FALLBACK_GBS = 6650.0


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), float(p.get("bf16_tflops", 1590.0)), float(p.get("bf16_tflops_sustained", 1400.0)), "measured"
    except Exception:
        return HBM_FALLBACK_GBS, 1590.0, 1400.0, "fallback"


# ------------------------------------------------------------------------------------------
class ClockSampler:
    """SM clocks and clock-event (throttle) reasons sampled DURING the timed region: an NVML
    thread every ~2 ms (the timed region of the default run is tens of ms, too short for
    nvidia-smi's 50 ms loop, which also starts ~100 ms late); nvidia-smi if NVML is missing."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, gpu_index, period_s=0.002):
        self.idx = gpu_index
        self.period = period_s
        self.p = None
        self.nv = None
        self.samples = []            # (sm_mhz, max_mhz, set(reasons))
        self.out = ""

    def _nvml_loop(self):
        import pynvml as N
        bits = {"hw_slowdown": N.nvmlClocksEventReasonHwSlowdown,
                "hw_thermal_slowdown": N.nvmlClocksEventReasonHwThermalSlowdown,
                "sw_thermal_slowdown": N.nvmlClocksEventReasonSwThermalSlowdown,
                "sw_power_cap": N.nvmlClocksEventReasonSwPowerCap}
        while not self.stop.is_set():
            try:
                sm = N.nvmlDeviceGetClockInfo(self.nv, N.NVML_CLOCK_SM)
                mx = N.nvmlDeviceGetMaxClockInfo(self.nv, N.NVML_CLOCK_SM)
                r = N.nvmlDeviceGetCurrentClocksEventReasons(self.nv)
                self.samples.append((float(sm), float(mx), {k for k, b in bits.items() if r & b}))
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        import threading
        try:
            import pynvml as N
            N.nvmlInit()
            self.nv = N.nvmlDeviceGetHandleByIndex(int(self.idx))
            self.stop = threading.Event()
            self.th = threading.Thread(target=self._nvml_loop, daemon=True)
            self.th.start()
            return self
        except Exception:
            self.nv = None
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.idx), f"--query-gpu={self.FIELDS}",
                                       "--format=csv,noheader,nounits", "-lms", "50"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.p = None
        return self

    def __exit__(self, *a):
        if self.nv is not None:
            self.stop.set()
            self.th.join(timeout=2)
            return
        if self.p is not None:
            self.p.terminate()
            try:
                self.out, _ = self.p.communicate(timeout=5)
            except Exception:
                self.p.kill()

    def summary(self):
        sm, mx, reasons = [], 0.0, set()
        for s_, m_, r_ in self.samples:
            sm.append(s_)
            mx = max(mx, m_)
            reasons |= r_
        for line in (self.out or "").splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = max(mx, float(f[2]))
            except ValueError:
                continue
            for nm, v in zip(self.NAMES, f[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        load = [s for s in sm if s > 300] or sm
        return {"sm_mhz": statistics.median(load) if load else None, "sm_max_mhz": mx or None,
                "reasons": sorted(reasons), "samples": len(sm),
                "source": "nvml" if self.nv is not None else "nvidia-smi"}


def physical_gpu_index(local_rank):
    vis = os.environ.get("CUDA_VISIBLE_DEVICES")
    if vis:
        ids = [v.strip() for v in vis.split(",") if v.strip()]
        if local_rank < len(ids) and ids[local_rank].isdigit():
            return int(ids[local_rank])
    return local_rank


# ------------------------------------------------------------------------------------------
def dist_setup(dry_run=False):
    """One process per GPU (torch.distributed.run sets RANK / WORLD_SIZE / LOCAL_RANK). At
    world > 1 the process group is initialised here, once, for every config: NCCL on the GPU box
    (it only carries the timing reductions and the job-queue bookkeeping: the path itself is
    replicas), gloo for --dry-run on CPU."""
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # FLEP_SHARE_GPU=1 (functional test of the N > 1 path on a one-GPU box): every rank uses the
    # visible GPUs round-robin and the process group runs on gloo (NCCL refuses a shared GPU);
    # the numbers of such a run are not scaling measurements
    share = os.environ.get("FLEP_SHARE_GPU") == "1"
    if world > 1:
        import torch
        import torch.distributed as dist
        if share and torch.cuda.is_available():
            local = local % max(1, torch.cuda.device_count())
        if not dist.is_initialized():
            if dry_run or share or not torch.cuda.is_available():
                dist.init_process_group("gloo")
            else:
                torch.cuda.set_device(local)
                dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    return rank, world, local


def allreduce_max(vals, world, torch):
    if world == 1:
        return vals
    import torch.distributed as dist
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor(vals, dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return t.tolist()


def allreduce_mean(vals, world, torch):
    if world == 1:
        return vals
    import torch.distributed as dist
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor(vals, dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return (t / world).tolist()


def gather_objects(obj, world):
    """Every rank's `obj` (host-side bookkeeping only), in rank order."""
    if world == 1:
        return [obj]
    import torch.distributed as dist
    out = [None] * world
    dist.all_gather_object(out, obj)
    return out


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        if dist.get_backend() == "nccl":
            import torch
            dist.barrier(device_ids=[torch.cuda.current_device()])
        else:
            dist.barrier()


def relaunch_under_torchrun(n):
    """`bench.py --gpus N` without a torchrun environment: re-execute this command as N ranks
    (one process per GPU, rendezvous on 127.0.0.1) and return their exit code."""
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


# ------------------------------------------------------------------------------------------
SPMV_ROWS = 1 << 20
STENCIL_N = 4096


def spmv_bytes(rowptr, rows, cols):
    nnz = int(rowptr[-1])
    return 8 * nnz + 8 * rows + 4 * cols      # 8 B/nnz + 8 B/row + 4 B/col


def stencil_bytes(n):
    return 8 * n * n                            # 8 B/cell


class Workload:
    def __init__(self, torch, seed_off=0):
        self.torch = torch
        self.rowptr, self.col, self.val, self.x = gen.csr_inputs(SPMV_ROWS, seed=2 + seed_off)
        self.st_in = gen.stencil_f32_input(STENCIL_N, seed=3 + seed_off)
        dev = "cuda"
        T = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(dev)  # noqa: E731
        self.d_rowptr, self.d_col, self.d_val, self.d_x = T(self.rowptr), T(self.col), T(self.val), T(self.x)
        self.d_y = torch.zeros(SPMV_ROWS, dtype=torch.float32, device=dev)
        self.d_in = T(self.st_in)
        self.d_out = torch.empty_like(self.d_in)
        self.nnz = int(self.rowptr[-1])
        self.spmv_bytes = spmv_bytes(self.rowptr, SPMV_ROWS, SPMV_ROWS)
        self.st_bytes = stencil_bytes(STENCIL_N)


class L2Flush:
    """Evict L2 between timed iterations: write a buffer of 2x the L2 size (the contract's flush),
    then read a second one so that the dirty lines the write left behind are written back by the
    flush itself and not by the next timed kernel."""

    def __init__(self, torch):
        l2 = torch.cuda.get_device_properties(0).L2_cache_size
        n = max(2 * l2, 256 << 20)
        self.w = torch.empty(n, dtype=torch.uint8, device="cuda")
        self.r = torch.zeros(n // 4, dtype=torch.int32, device="cuda")
        self.out = torch.zeros((), dtype=torch.int64, device="cuda")
        self.torch = torch

    def zero_(self):
        self.w.zero_()
        self.r.sum()


def l2_flush_buffer(torch):
    return L2Flush(torch)


def run_temporal(args, rank, world, local):
    import torch
    from paper_conf_asplos_wulzj17_b200 import flep as F
    torch.cuda.set_device(local)
    hbm, _, _, peak_src = peaks()
    wl = Workload(torch)
    flush = l2_flush_buffer(torch)
    # The waiting kernel is enqueued right behind the victim so that it is already pending when
    # the request fires. The victim's stream gets the higher CUDA priority only so that the
    # hardware dispatches all victim workers first when both become ready together (checked
    # per step: the waiting kernel must not start before the request).
    A = torch.cuda.Stream(priority=-2)
    B = torch.cuda.Stream(priority=0)
    rt = F.Runtime(device=local, exec_on_user_stream=True)
    num_sms = rt.num_sms
    # the victim fetches speculatively (R34): poll and fetch in one round trip, a fetched chunk is
    # returned through the worker's record on a stop
    kLP = rt.register_kernel(F.BODY_SPMV_CSR_F32, chunk=args.lp_chunk, poll=args.lp_poll, name="spmv",
                             prefetch=bool(args.prefetch), spec_fetch=bool(args.lp_spec), ctas_per_sm=args.lp_cps)
    # the waiting (high-priority) kernel is never preempted here: it is tuned for throughput (CLC
    # task fetch, C = 1, K = 4: 4.6 % over the unwrapped grid vs 19 % for the counter worker,
    # profiles/r01_bench_clc.json), the victim for latency (atomic counter, C = K = 1)
    kHP = rt.register_kernel(F.BODY_STENCIL5_F32, chunk=args.hp_chunk, poll=args.hp_poll, name="stencil",
                             prefetch=bool(args.hp_prefetch), async_poll=bool(args.hp_async),
                             clc=bool(args.hp_clc))
    lp_args = F.spmv_args(wl.d_y, wl.d_rowptr, wl.d_col, wl.d_val, wl.d_x)
    hp_args = F.stencil_args(wl.d_out, wl.d_in)
    lp_grid, hp_grid = F.spmv_grid(SPMV_ROWS), F.stencil_grid(STENCIL_N)
    n_lp = lp_grid[0]
    g = gen.rng(1000 + rank)

    def step(k_lp=None):
        k_lp = kLP if k_lp is None else k_lp
        tstar = int(g.integers(n_lp // 4, 3 * n_lp // 4))
        with torch.cuda.stream(A):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True)
            e0.record(A)
        rt.arm_next_trigger(tstar, num_sms)
        h_lp = rt.launch(k_lp, lp_grid, lp_args, priority=0, stream=A)
        B.wait_event(e0)
        h_hp = rt.launch(kHP, hp_grid, hp_args, priority=1, stream=B)
        rt.wait_epoch(h_lp, timeout_ns=10_000_000_000)
        info = rt.query(h_lp)
        preempted = info.state == F.STATE_PREEMPTED
        rt.sync(h_hp, timeout_ns=10_000_000_000)      # FLEP resumes the victim when the HP ends
        if preempted:
            rt.resume(h_lp)
        rt.sync(h_lp, timeout_ns=10_000_000_000)
        e_b = torch.cuda.Event()
        e_b.record(B)
        A.wait_event(e_b)
        e1 = torch.cuda.Event(enable_timing=True)
        e1.record(A)
        e1.synchronize()
        ep = rt.epoch_info(h_lp, 1)
        hp_ev = rt.events(h_hp, 1)
        lp_ev = rt.events(h_lp, 1)
        t_req = ep.t_trigger
        hp_start = min(e.t_entry for e in hp_ev)
        hp_end = max(e.t_exit for e in hp_ev)
        lp_start = min(e.t_entry for e in lp_ev)
        launches = rt.query(h_lp).epoch + rt.query(h_hp).epoch
        valid = preempted and t_req > 0 and hp_start >= t_req
        return {
            "preempted": valid,
            "hp_started_early": bool(t_req and hp_start < t_req),
            "latency_us": (hp_start - t_req) / 1e3 if t_req else None,
            "drain_us": (ep.t_end - t_req) / 1e3 if t_req else None,
            "hp_turnaround_us": (hp_end - t_req) / 1e3 if t_req else None,
            "lp_before_request_us": (t_req - lp_start) / 1e3 if t_req else None,
            "step_ms": e0.elapsed_time(e1),
            "launches": launches,
            "tstar": tstar,
        }

    res = []
    with ClockSampler(physical_gpu_index(local)) as clk:
        for _ in range(args.warmup):
            step()
        torch.cuda.synchronize()
        barrier(world)
        t_start = time.perf_counter()
        for _ in range(args.steps):
            res.append(step())
        torch.cuda.synchronize()
        barrier(world)
        wall = time.perf_counter() - t_start
    clocks = clk.summary()
    # correctness spot check of the last co-run (device result vs NumPy fp64 rows / cells sampled)
    parity = spot_parity(wl, torch)

    lat = [r["latency_us"] for r in res if r["preempted"]]
    drain = [r["drain_us"] for r in res if r["preempted"]]
    hpt = [r["hp_turnaround_us"] for r in res if r["preempted"]]
    ms = [r["step_ms"] for r in res]
    p50 = float(np.median(lat)) if lat else float("nan")
    p99 = float(np.percentile(lat, 99)) if lat else float("nan")
    ms_step = float(np.mean(ms))
    d50 = float(np.median(drain)) if drain else float("nan")
    red = allreduce_max([d50, ms_step, p50], world, torch)

    # ---- wrapper overhead + roofline (standalone launches, L2 flushed, CUDA events on stream A)
    kern = kernel_timings(rt, F, torch, wl, flush, A, kLP, kHP, lp_args, hp_args, lp_grid, hp_grid, args.reps)
    dom = max(("spmv", "stencil"), key=lambda k: kern[k]["wrapped_us"])
    algo = wl.spmv_bytes if dom == "spmv" else wl.st_bytes
    achieved = algo / (kern[dom]["wrapped_us"] * 1e-6) / 1e9
    prof_traffic = load_traffic(dom)
    # The SpMV's algorithmic bytes stream at a fraction of HBM speed because its x[col[p]] gathers
    # are random 4-B reads of an L2-resident vector: one 32-B sector request per nonzero. Its real
    # ceiling is the measured random-gather rate (probes/probe6.cu: same x size and nnz).
    # latency budget: the drain against one chunk of the victim (a worker stops at
    # its next poll, i.e. after the chunk it is running: at C = K = 1 the drain is bounded by one
    # chunk's execution time plus the exit), with the chunk time from the standalone wrapped run
    _, w_lp = rt.workers_for(F.BODY_SPMV_CSR_F32)
    if args.lp_cps:
        w_lp = min(w_lp, args.lp_cps * num_sms)
    chunk_us = kern["spmv"]["wrapped_us"] * w_lp * args.lp_chunk / n_lp
    latency_budget = {"drain_p50_us": round(d50, 3), "victim_chunk_us": round(chunk_us, 3),
                      "drain_over_chunk": round(d50 / chunk_us, 3) if chunk_us else None,
                      "definition": "victim chunk time = standalone wrapped SpMV time x W x C / N (each of "
                                    "the W workers runs N/(W C) chunks back to back)",
                      "kernel_boundary_us": 2.36, "kernel_boundary_source": "profiles/r01_probe_exit_accounting.jsonl (empty grid, back to back)"}
    gpk = load_gather_peak()
    g_ach = wl.nnz / (kern["spmv"]["wrapped_us"] * 1e-6)
    gather_roofline = {"bound": "l1_gather", "kernel": "flep_worker<spmv>", "achieved": float(f"{g_ach:.4g}"),
                       "peak": gpk, "unit": "gathers/s", "frac": round(g_ach / gpk, 4) if gpk else None,
                       "unwrapped_frac": round(wl.nnz / (kern["spmv"]["unwrapped_us"] * 1e-6) / gpk, 4) if gpk else None,
                       "peak_source": "measured: probes/probe6.cu (profiles/r0[12]_probe_gather_ceiling.jsonl)",
                       "limiter": "L1TEX->XBAR miss-request interface (one request per cycle per SM): probe 6 runs it at 83 % "
                                  "of peak (elapsed), the SpMV worker at 61 %, unwrapped 67 % (profiles/r02_probe6_limiter.json, "
                                  "r02_ncu_full_summary.json); every x gather that misses L1 (95 %) is one request"}
    roofline = {"bound": "hbm", "achieved": round(achieved, 1), "peak": hbm, "unit": "GB/s",
                "frac": round(achieved / hbm, 4), "traffic": prof_traffic, "kernel": f"flep_worker<{dom}>",
                "algorithmic_bytes": algo, "peak_source": peak_src}

    # the throughput operating point of the same co-run (SURVEY §8(d) "(C, K) sweep"): the victim
    # fetches C = 2 blocks per atomic, so its drain is up to two blocks and its overhead is paid
    # per 256 rows; measured with the same steps, the same kernel timing protocol
    op2 = None
    if args.lp_chunk == 1 and args.op2:
        kLP2 = rt.register_kernel(F.BODY_SPMV_CSR_F32, chunk=2, poll=args.lp_poll, name="spmv-c2",
                                  spec_fetch=bool(args.lp_spec), ctas_per_sm=args.lp_cps)
        for _ in range(args.warmup):
            step(kLP2)
        r2 = [step(kLP2) for _ in range(args.steps)]
        d2 = [r["drain_us"] for r in r2 if r["preempted"]]
        kt2 = kernel_timings(rt, F, torch, wl, flush, A, kLP2, kHP, lp_args, hp_args, lp_grid, hp_grid, args.reps,
                             only=("spmv",))
        op2 = {"lp_chunk": 2, "drain_us": {"p50": round(float(np.median(d2)), 3) if d2 else None,
                                           "p99": round(float(np.percentile(d2, 99)), 3) if d2 else None,
                                           "max": round(max(d2), 3) if d2 else None, "preempted_steps": len(d2)},
               "spmv": kt2["spmv"]}
    e2e = run_e2e(F, torch, wl, local, args.e2e_steps, args)
    _diag = run_e2e(F, torch, wl, local, args.e2e_steps, args, diag=True)
    e2e["breakdown_us_p50"] = _diag.get("breakdown_us_p50")
    e2e["breakdown_steps"] = _diag.get("diag_points")
    rt.close()

    out = {
        "metric": METRIC,
        "value": round(red[0], 3),
        "unit": "us",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": round(red[1], 4),
        "higher_is_better": False,
        "scaling": "weak",
        "vs_baseline": None,
        "dtype": "f32",
        "data": "synthetic (seeded; synth/gen.py)",
        "config": {"workload": "configs[1]: full-GPU temporal preemption of SpMV-CSR fp32 (2^20 rows, "
                               f"{wl.nnz} nnz, low priority) by stencil5 fp32 4096^2 (high priority)",
                   "lp_chunk": args.lp_chunk, "lp_poll": args.lp_poll, "hp_chunk": args.hp_chunk, "hp_poll": args.hp_poll, "hp_clc": bool(args.hp_clc), "hp_prefetch": bool(args.hp_prefetch),
                   "hp_async_poll": bool(args.hp_async),
                   "prefetch": bool(args.prefetch), "lp_spec_fetch": bool(args.lp_spec),
                   "lp_ctas_per_sm": args.lp_cps or w_lp // num_sms,
                   "flag": "stream_memop (device self-trigger for the request)",
                   "l2": "flushed between steps (write of 2x L2 bytes)", "parallelism": f"replicas x{world}"},
        "value_definition": "full-GPU preemption latency (device %globaltimer): request visible on the GPU -> "
                            "last victim CTA gone (all 148 SMs released), p50 over the timed steps, max over ranks",
        "waiting_start_us": {"p50": round(red[2], 3), "p99": round(p99, 3), "max": round(max(lat), 3) if lat else None,
                             "min": round(min(lat), 3) if lat else None, "preempted_steps": len(lat),
                             "definition": "request visible on the GPU -> first CTA of the (already pending) waiting kernel running"},
        "drain_us": {"p50": round(d50, 3), "p99": round(float(np.percentile(drain, 99)), 3) if drain else None,
                     "max": round(max(drain), 3) if drain else None},
        "hp_turnaround_us": {"p50": round(float(np.median(hpt)), 3) if hpt else None},
        "target_20us_met": bool(drain) and max(drain) < 20.0,
        "latency_budget": latency_budget,
        "wrapper_overhead_pct": {k: v["overhead_pct"] for k, v in kern.items()},
        "operating_points": {"latency (victim C = 1, the headline)": {
                                 "lp_chunk": args.lp_chunk, "drain_us_p50": round(d50, 3),
                                 "spmv_overhead_pct": kern["spmv"]["overhead_pct"],
                                 "spmv_overhead_pct_ci95": kern["spmv"].get("overhead_pct_ci95")},
                             "throughput (victim C = 2)": op2},
        "kernels": kern,
        "roofline": roofline,
        "gather_roofline": gather_roofline,
        "e2e": e2e,
        "gpu_launches": int(sum(r["launches"] for r in res)),
        "hp_started_before_request": int(sum(1 for r in res if r["hp_started_early"])),
        "clocks": clocks,
        "parity": parity,
        "wall_s_timed": round(wall, 3),
    }
    if rank == 0:
        out["cpu_baseline"] = cpu_baseline(wl)
    del wl, flush
    torch.cuda.empty_cache()
    if args.sub:
        subs = sub_records(args, rank, world, local)
        if rank == 0:
            out["configs"] = subs
    if rank == 0:
        print(json.dumps(out), flush=True)
    barrier(world)


def spot_parity(wl, torch):
    """Sampled element-by-element check of the last co-run's outputs (bench_check: NumPy fp64)."""
    import bench_check as BC
    g = gen.rng(7)
    rows = g.integers(0, SPMV_ROWS, 512)
    y = wl.d_y.cpu().numpy()
    worst = 0.0
    for r in rows:
        s, e = wl.rowptr[r], wl.rowptr[r + 1]
        ref, absum = BC.spmv_row(wl.col[s:e], wl.val[s:e], wl.x)
        d = max(abs(ref), absum, 1e-30)
        worst = max(worst, abs(float(y[r]) - ref) / d)
    out = wl.d_out.cpu().numpy()
    ref, absum = BC.stencil5_f32(wl.st_in[:130, :130])
    d = np.maximum(np.abs(ref), absum)
    worst_st = float(np.max(np.abs(out[:129, :129] - ref[:129, :129]) / np.where(d[:129, :129] > 0, d[:129, :129], 1)))
    return {"spmv_max_rel": worst, "stencil_max_rel": worst_st, "tol": 1e-5,
            "ok": bool(worst <= 1e-5 and worst_st <= 1e-5)}


def kernel_timings(rt, F, torch, wl, flush, A, kLP, kHP, lp_args, hp_args, lp_grid, hp_grid, reps,
                   only=("spmv", "stencil")):
    res = {}
    for name, k, body, a, grid, nbytes in (("spmv", kLP, F.BODY_SPMV_CSR_F32, lp_args, lp_grid, wl.spmv_bytes),
                                           ("stencil", kHP, F.BODY_STENCIL5_F32, hp_args, hp_grid, wl.st_bytes)):
        if name not in only:
            continue
        tw, tu = [], []
        for r in range(reps + 2):
            for mode in ("w", "u"):
                with torch.cuda.stream(A):
                    flush.zero_()
                    dither(torch)
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(A)
                if mode == "w":
                    h = rt.launch(k, grid, a, stream=A)
                else:
                    rt.launch_unwrapped(body, grid, a, stream=A)
                e1.record(A)
                e1.synchronize()
                if mode == "w":
                    rt.sync(h)
                if r >= 2:
                    (tw if mode == "w" else tu).append(e0.elapsed_time(e1) * 1e3)
        w_us, u_us = event_mean_us(tw), event_mean_us(tu)
        # 95 % confidence half-width of the overhead ratio (delta method on the sample means)
        aw, au = np.asarray(tw), np.asarray(tu)
        mw, mu = float(aw.mean()), float(au.mean())
        var_r = aw.var(ddof=1) / len(aw) / mu ** 2 + mw ** 2 * au.var(ddof=1) / len(au) / mu ** 4
        res[name] = {"stat": "trimmed mean (middle 80 %) of dithered CUDA-event durations",
                     "overhead_pct_mean": round((mw / mu - 1.0) * 100.0, 2),
                     "overhead_pct_ci95": round(1.96 * float(np.sqrt(var_r)) * 100.0, 2),
                     "samples": [len(tw), len(tu)],
                     "wrapped_us": round(w_us, 3), "unwrapped_us": round(u_us, 3),
                     "wrapped_min_us": round(min(tw), 3), "unwrapped_min_us": round(min(tu), 3),
                     "wrapped_gbs": round(nbytes / (w_us * 1e-6) / 1e9, 1),
                     "unwrapped_gbs": round(nbytes / (u_us * 1e-6) / 1e9, 1),
                     "overhead_pct": round((w_us / u_us - 1.0) * 100.0, 2),
                     "algorithmic_bytes": nbytes}
    return res


def load_gather_peak():
    """Measured random-gather ceiling (gathers/s) of probes/probe6.cu, committed under profiles/."""
    best = None
    for name in ("r01_probe_gather_ceiling.jsonl", "r02_probe6_gather_ceiling.jsonl"):
        try:
            with open(os.path.join(ROOT, "profiles", name)) as f:
                v = max(json.loads(l)["gathers_per_s"] for l in f if l.strip())
            best = v if best is None else max(best, v)
        except Exception:
            pass
    return best


def load_traffic(dom):
    """dram bytes per launch from the committed ncu --set full capture, if present."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        with open(p) as f:
            return json.load(f).get(dom)
    except Exception:
        return None


def run_e2e(F, torch, wl, local, steps, args, diag=False):
    """Same metric through the managed public API (HPF policy), with host buffers: every step
    copies the inputs from pinned host memory, the HP arrival is an intercepted flep_launch that
    makes the runtime preempt the running LP, and the outputs are read back. Latency = host
    clock from the runtime's preemption request to its observation of the drained epoch."""
    rt = F.Runtime(device=local, policy=F.POLICY_HPF, keep_logs=diag)
    kLP = rt.register_kernel(F.BODY_SPMV_CSR_F32, chunk=args.lp_chunk, poll=args.lp_poll, name="spmv",
                             model=(0, 0, 0, 0, 70_000), prefetch=bool(args.prefetch), started_hint=True,
                             host_relay=bool(args.e2e_relay), spec_fetch=bool(args.lp_spec), ctas_per_sm=args.lp_cps)
    kHP = rt.register_kernel(F.BODY_STENCIL5_F32, chunk=args.hp_chunk, poll=args.hp_poll, name="stencil",
                             model=(0, 0, 0, 0, 30_000), prefetch=bool(args.hp_prefetch), async_poll=bool(args.hp_async),
                             clc=bool(args.hp_clc))
    pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()  # noqa: E731
    h_rp, h_col, h_val, h_x, h_in = pin(wl.rowptr), pin(wl.col), pin(wl.val), pin(wl.x), pin(wl.st_in)
    h_y = torch.empty(SPMV_ROWS, dtype=torch.float32).pin_memory()
    h_out = torch.empty_like(h_in).pin_memory()
    A = torch.cuda.Stream(priority=0)
    B = torch.cuda.Stream(priority=-2)
    lp_args = F.spmv_args(wl.d_y, wl.d_rowptr, wl.d_col, wl.d_val, wl.d_x)
    hp_args = F.stencil_args(wl.d_out, wl.d_in)
    h2d = sum(t.numel() * t.element_size() for t in (h_rp, h_col, h_val, h_x, h_in))
    d2h = h_y.numel() * 4 + h_out.numel() * 4
    lats, step_ms, pre, parts, dev = [], [], 0, [], []
    for i in range(steps + 2):
        t0 = time.perf_counter()
        with torch.cuda.stream(A):
            for d, h in ((wl.d_rowptr, h_rp), (wl.d_col, h_col), (wl.d_val, h_val), (wl.d_x, h_x)):
                d.copy_(h, non_blocking=True)
        with torch.cuda.stream(B):
            wl.d_in.copy_(h_in, non_blocking=True)
        A.synchronize()
        if not args.e2e_overlap_copy:
            B.synchronize()    # both inputs resident: no DMA runs beside the co-run
        h_lp = rt.launch(kLP, F.spmv_grid(SPMV_ROWS), lp_args, priority=0, stream=A)
        t_w = time.perf_counter()
        while rt.query(h_lp).started_epoch < 1 and time.perf_counter() - t_w < 1.0:
            pass                                   # the HP arrives while the LP is running
        t_started_seen = F.now_ns()
        t_l0 = F.now_ns()
        h_hp = rt.launch(kHP, F.stencil_grid(STENCIL_N), hp_args, priority=1, stream=B)
        t_l1 = F.now_ns()
        ev = []
        rt.sync(h_hp, timeout_ns=10_000_000_000)
        rt.sync(h_lp, timeout_ns=10_000_000_000)
        with torch.cuda.stream(A):
            h_y.copy_(wl.d_y, non_blocking=True)
        with torch.cuda.stream(B):
            h_out.copy_(wl.d_out, non_blocking=True)
        A.synchronize()
        B.synchronize()
        dt = (time.perf_counter() - t0) * 1e3
        info = rt.query(h_lp)
        if diag and info.epoch >= 2:  # the victim's first-epoch worker log, kept (keep_logs): read
            ev = rt.events(h_lp, 1)   # after the step, so the host thread waits in flep_sync as usual
        if i >= 2:
            step_ms.append(dt)
            if info.epoch >= 2 and info.t_last_drain > 0:
                pre += 1
                lats.append((info.t_last_drain - info.t_last_request) / 1e3)
                parts.append(((info.t_last_request - t_l0) / 1e3, (t_l1 - info.t_last_request) / 1e3))
                # device <-> host clock: worker 0 publishes "started" right after stamping t_entry,
                # and the host saw it at t_started_seen (offset error: one PCIe write + a poll)
                w0 = [e for e in ev if e.t_entry > 0]
                if w0:
                    off = t_started_seen - min(e.t_entry for e in w0)      # host - device
                    ys = [e.t_exit for e in ev if e.reason == F.REASON_YIELD]
                    if ys:
                        dev.append(((min(ys) + off - info.t_last_request) / 1e3,
                                    (max(ys) - min(ys)) / 1e3,
                                    (info.t_last_drain - (max(ys) + off)) / 1e3))
    dec = rt.decision_log()
    rt.close()
    return {"value": round(float(np.median(lats)), 3) if lats else None, "unit": "us",
            "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
            "preempted_steps": pre, "steps": steps, "ms_per_step": round(float(np.median(step_ms)), 3),
            "definition": "host clock: HPF runtime's preemption request (cuStreamWriteValue32 issued) -> "
                          "host observes the victim's drained epoch; inputs H2D from pinned memory (both "
                          "copies complete before the victim starts) and outputs D2H inside every step",
            "note": "the victim uses the request-relay CTA (R28): without it a stream memop issued while a "
                    "large H2D copy is in flight reaches the GPU ~20 us later (39 us with the waiting "
                    "kernel's 67 MB input copy overlapping the co-run vs 19.6 us with the relay)",
            "relay": bool(args.e2e_relay), "overlap_copy": bool(args.e2e_overlap_copy),
            "decisions_last": [F.ACTION_NAMES[d[1]] for d in dec[-4:]],
            "host_path_us_p50": {"launch_call_to_request": round(float(np.median([a for a, _ in parts])), 3) if parts else None,
                                 "request_to_launch_return": round(float(np.median([b for _, b in parts])), 3) if parts else None},
            "diag_points": [len(dev), pre],
            "breakdown_us_p50": ({"request_to_first_yield": round(float(np.median([a for a, _, _ in dev])), 3),
                                  "yield_spread": round(float(np.median([b for _, b, _ in dev])), 3),
                                  "last_yield_to_host_seen": round(float(np.median([c for _, _, c in dev])), 3),
                                  "note": "device times mapped to the host clock through the started hint: "
                                          "the host sees that hint one PCIe write + one poll late, so every "
                                          "mapped device time reads late by that much (the last leg can read "
                                          "negative); the logs are read after the step (keep_logs)"} if dev else None)}


def cpu_baseline(wl):
    """The oracle (as it stands) on the host cores, on this workload: a non-preemptive CPU
    program must finish the LP's remaining blocks before the HP can start, so its 'preemption
    latency' is the oracle time for the LP rows after t* (t* = N/2 here)."""
    from oracle import workloads as W
    half = SPMV_ROWS // 2
    s = wl.rowptr[half]
    rp = (wl.rowptr[half:] - s).astype(np.int32)
    t0 = time.perf_counter()
    W.spmv_csr(rp, wl.col[s:], wl.val[s:], wl.x)
    t_rem = time.perf_counter() - t0
    t0 = time.perf_counter()
    W.stencil5_f32(wl.st_in)
    t_st = time.perf_counter() - t0
    return {"value": round(t_rem * 1e6, 1), "unit": "us", "cores": 1, "kind": "oracle",
            "sample": "oracle SpMV over the LP's remaining half (2^19 rows) = the HP's wait on a "
                      f"non-preemptive CPU; oracle stencil 4096^2 alone took {t_st * 1e6:.0f} us",
            "threads_note": "numpy element-wise + np.add.at, single-threaded"}


def run_reference(args, rank, world):
    """--impl reference: the oracle, timed on the host cores, same config/metric/unit. A step is
    what a non-preemptive program makes the waiting kernel wait for: the oracle SpMV over the LP
    rows after a seeded block t*. `ms_per_step` is the mean of exactly those timed steps."""
    if rank != 0:
        return
    from oracle import workloads as W
    rowptr, col, val, x = gen.csr_inputs(SPMV_ROWS, seed=2)
    from paper_conf_asplos_wulzj17_b200.flep import SPMV_ROWS_PER_BLOCK
    n_lp = (SPMV_ROWS + SPMV_ROWS_PER_BLOCK - 1) // SPMV_ROWS_PER_BLOCK
    g = gen.rng(1000)
    lats = []
    for i in range(args.warmup + args.steps):
        tstar = int(g.integers(n_lp // 4, 3 * n_lp // 4))
        r0 = tstar * SPMV_ROWS_PER_BLOCK
        s = rowptr[r0]
        t0 = time.perf_counter()
        W.spmv_csr((rowptr[r0:] - s).astype(np.int32), col[s:], val[s:], x)
        t1 = time.perf_counter()
        if i >= args.warmup:
            lats.append((t1 - t0) * 1e6)
    v = float(np.median(lats))
    extra = oracle_timings()
    out = {"impl": "reference", "metric": METRIC, "value": round(v, 1), "unit": "us", "n_gpus": world,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(float(np.mean(lats)) / 1e3, 3),
           "higher_is_better": False, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
           "data": "synthetic (seeded; synth/gen.py)",
           "config": {"workload": "configs[1]: full-GPU temporal preemption of SpMV-CSR fp32 (2^20 rows) by stencil5 "
                                  "fp32 4096^2 -- CPU oracle arm: the HP waits for the LP's remaining rows"},
           "cpu_baseline": {"value": round(v, 1), "unit": "us", "cores": 1, "kind": "oracle",
                            "sample": "per step: oracle SpMV over the LP rows after a seeded t* (what a "
                                      "non-preemptive program must finish before the HP starts); ms_per_step is the "
                                      "mean of these timed steps"},
           "e2e": {"value": round(v, 1), "unit": "us", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
           "oracle_timings": extra}
    print(json.dumps(out), flush=True)


def oracle_timings():
    """SURVEY §8(d) oracle-timing protocol beside the reference arm: the host (model, cores, BLAS
    threads), the fp64 GEMM oracle on a bounded sample (2048^3, all cores; 8192^3 extrapolated by
    the flop ratio) and the DES per trace (configs[3]: 64 kernels, configs[4]: 512)."""
    import platform
    from oracle import des, workloads as W
    info = {"cpu_count": os.cpu_count(), "machine": platform.machine()}
    try:
        with open("/proc/cpuinfo") as fh:
            info["cpu_model"] = next((l.split(":", 1)[1].strip() for l in fh if l.startswith("model name")), None)
    except OSError:
        info["cpu_model"] = None
    try:
        from threadpoolctl import threadpool_info
        info["blas"] = [{"api": d.get("internal_api"), "threads": d.get("num_threads")} for d in threadpool_info()]
    except Exception:
        info["blas"] = None
    a_bits, b_bits = gen.gemm_bf16_inputs(2048, 2048, 2048, seed=60)
    t0 = time.perf_counter()
    W.gemm_bf16(a_bits, b_bits)
    t_g = time.perf_counter() - t0
    info["gemm_fp64_2048cubed_s"] = round(t_g, 3)
    info["gemm_fp64_8192cubed_s_extrapolated"] = round(t_g * 64, 2)
    for name, n in (("configs[3]", 64), ("configs[4]", 512)):
        tr = gen.queue_trace(5 if n == 64 else 6, n, 200_000)
        ks = [des.KernelSpec(j["id"], j["arrival_ns"], 0, 100_000 * (1 + j["size_class"] * 10), 20_000,
                             100_000 * (1 + j["size_class"] * 10)) for j in tr]
        t0 = time.perf_counter()
        des.simulate(des.HPF, ks)
        info[f"des_hpf_{name}_{n}_kernels_ms"] = round((time.perf_counter() - t0) * 1e3, 2)
    return info


def sub_records(args, rank, world, local):
    """The other BASELINE configs as sub-records of the default line (each with its own clocks):
    configs[0] (SAXPY-int co-run, exactness), configs[2] (spatial yield per width: the manual
    device-triggered sweep and the managed spatial-HPF decision path, victim checked against a
    NumPy reference), configs[3] (64-kernel same-priority queue: ANTT/STP, decision logs),
    configs[4] (one 512-kernel job queue over the N GPUs of this run), E13 (never-preempted
    overhead of FLEP vs kernel slicing) and the co-run matrices (E4 / E6 / E8: Figs. 8,
    10, 12)."""
    import copy
    import bench_configs as BCF
    a = copy.copy(args)
    a.sub_record = True
    a.steps, a.warmup = args.sub_steps, 3
    out, timing = {}, {}
    for name, fn in (("configs[0]", BCF.run_corun1), ("configs[2]", BCF.run_spatial),
                     ("configs[2]_managed", BCF.run_spatial_managed), ("configs[3]", BCF.run_queue),
                     ("configs[4]", BCF.run_scale_queue), ("E13_never_preempted", BCF.run_slicing_overhead),
                     ("coruns_E4_E6_E8", BCF.run_coruns)):
        if name in args.skip_sub:
            continue
        t0 = time.perf_counter()
        r = fn(a, rank, world, local)
        timing[name] = round(time.perf_counter() - t0, 1)
        if rank == 0 and r is not None:
            for k in ("metric", "n_gpus", "higher_is_better", "scaling", "vs_baseline", "data"):
                r.pop(k, None)
            out[name] = r
    if rank == 0:
        out["wall_s"] = timing
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="flep", choices=["flep", "reference"])
    ap.add_argument("--config", default="temporal", choices=["temporal", "corun1", "spatial", "spatial_managed", "queue",
                                                             "scale", "ffs", "model", "gemm", "tune", "clc", "delay",
                                                             "spatial_f1", "slicing", "coruns"])
    ap.add_argument("--corun-reps", type=int, default=3, help="config coruns: runs per case and policy")
    ap.add_argument("--dry-run", action="store_true",
                    help="configs[4] launcher and control flow without CUDA (CPU, gloo); one JSON line")
    ap.add_argument("--sub", type=int, default=1, help="default run: add the configs[0,2,3,4] sub-records")
    ap.add_argument("--op2", type=int, default=1, help="default run: also measure the C = 2 operating point")
    ap.add_argument("--sub-steps", type=int, default=12, help="timed trials per sub-record case")
    ap.add_argument("--skip-sub", default="", help="comma list of sub-record names to skip")
    ap.add_argument("--scale-kernels", type=int, default=512)
    ap.add_argument("--model-train", type=int, default=100)
    ap.add_argument("--model-test", type=int, default=30)
    ap.add_argument("--overhead-runs", type=int, default=50)
    ap.add_argument("--ffs-seconds", type=float, default=1.0)
    ap.add_argument("--corun-cps", type=int, default=2)
    ap.add_argument("--queue-kernels", type=int, default=64)
    ap.add_argument("--rho", type=float, default=1.0)
    ap.add_argument("--lp-chunk", type=int, default=1)
    ap.add_argument("--prefetch", type=int, default=0)
    ap.add_argument("--hp-chunk", type=int, default=1)
    ap.add_argument("--hp-poll", type=int, default=4)
    ap.add_argument("--hp-clc", type=int, default=1, help="waiting kernel: CLC task fetch (R25)")
    ap.add_argument("--hp-prefetch", type=int, default=0)
    ap.add_argument("--hp-async", type=int, default=0, help="waiting kernel: async poll (R22)")
    ap.add_argument("--lp-poll", type=int, default=1)
    ap.add_argument("--lp-spec", type=int, default=1, help="victim: speculative fetch (R34)")
    ap.add_argument("--lp-cps", type=int, default=0, help="victim: resident workers per SM (0 = occupancy, P:128)")
    ap.add_argument("--reps", type=int, default=40)
    ap.add_argument("--e2e-relay", type=int, default=1, help="e2e victim with the request-relay CTA (R28)")
    ap.add_argument("--e2e-overlap-copy", type=int, default=0, help="e2e: let the HP's input copy overlap the co-run")
    ap.add_argument("--e2e-steps", type=int, default=10)
    ap.add_argument("--tune-bound", type=float, default=0.04, help="config tune: overhead bound (P:166: 4 %%)")
    ap.add_argument("--gemm-in-tile", type=int, default=1, help="config gemm: in-tile preemption (1) or tile granularity (0)")
    ap.add_argument("--gemm-pair", type=int, default=0, help="config gemm: the 1-CTA body (0), the CTA-pair body (1) or its 256x512 tile (2)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    args.skip_sub = [x.strip() for x in args.skip_sub.split(",") if x.strip()]
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(relaunch_under_torchrun(args.gpus))
    rank, world, local = dist_setup(dry_run=args.dry_run)
    if world != args.gpus and rank == 0:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}; using {world} ranks", file=sys.stderr)
    if args.dry_run:
        import bench_configs
        bench_configs.run_scale_dry(args, rank, world, local)
        return
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    from paper_conf_asplos_wulzj17_b200 import build
    if rank == 0:
        build.build()
    if world > 1:
        barrier(world)                       # rank 0's build (if any) is complete
    if args.config == "temporal":
        run_temporal(args, rank, world, local)
    else:
        import bench_configs
        fn = {"spatial": bench_configs.run_spatial, "spatial_managed": bench_configs.run_spatial_managed,
              "corun1": bench_configs.run_corun1, "gemm": bench_configs.run_gemm_preempt,
              "tune": bench_configs.run_tune, "ffs": bench_configs.run_ffs, "model": bench_configs.run_model,
              "clc": bench_configs.run_clc, "delay": bench_configs.run_delay,
              "spatial_f1": bench_configs.run_spatial_f1, "queue": bench_configs.run_queue,
              "scale": bench_configs.run_scale_queue, "slicing": bench_configs.run_slicing_overhead,
              "coruns": bench_configs.run_coruns}[args.config]
        fn(args, rank, world, local)


if __name__ == "__main__":
    main()
