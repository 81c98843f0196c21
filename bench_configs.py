"""Additional bench.py configurations (BASELINE.json configs[0], [2], [3], [4]).

Each function prints one JSON line in the same contract shape as the default run; `value` is the
configuration's headline (stated in `value_definition`). All device times come from the
workers' %globaltimer event log; all inputs are seeded (synth/gen.py)."""
from __future__ import annotations

import json
import os
import time

import numpy as np

from synth import gen

METRIC = ("preemption latency µs (full vs N-SM yield); wrapper overhead % of HBM/tensor roofline; "
          "co-run NATT")


def _emit(out, rank, args):
    """Print the config's JSON line (rank 0) when it runs as bench.py's --config; as a sub-record
    of the default run (args.sub_record) it is only returned."""
    if rank == 0 and not getattr(args, "sub_record", False):
        print(json.dumps(out), flush=True)


def _span(evs):
    return min(e.t_entry for e in evs), max(e.t_exit for e in evs)


# ------------------------------------------------------------------------------------------
def run_spatial(args, rank, world, local):
    """configs[2]: spatial preemption yielding n in {8,16,32,74} of 148 SMs (and 148 = temporal
    reference) to a small waiting kernel while a 2D 5-point stencil (16384^2) keeps running.
    Paper metric: overhead = (T_FLEP - T_org) / T_org, T_org = victim then waiting kernel
    back to back (no preemption); reduction vs temporal (Fig. 15)."""
    import torch
    from bench import ClockSampler, L2Flush, barrier, physical_gpu_index
    from paper_conf_asplos_wulzj17_b200 import flep as F
    torch.cuda.set_device(local)
    rt = F.Runtime(device=local, exec_on_user_stream=True)
    n_st = 16384
    g = torch.Generator(device="cuda")
    g.manual_seed(4 + rank)
    v_in = torch.rand(n_st, n_st, device="cuda", generator=g)
    v_out = torch.empty_like(v_in)
    k_v = rt.register_kernel(F.BODY_STENCIL5_F32, chunk=1, poll=1, name="victim")
    k_w = rt.register_kernel(F.BODY_SAXPY_F32, chunk=1, poll=1, name="waiting")
    cps_w, _ = rt.workers_for(F.BODY_SAXPY_F32)
    widths = [8, 16, 32, 74, rt.num_sms]
    n_max = max(widths) * cps_w * 256
    wx = torch.rand(n_max, device="cuda", generator=g)
    wy = torch.rand(n_max, device="cuda", generator=g)
    flush = L2Flush(torch)
    A = torch.cuda.Stream(priority=-2)
    B = torch.cuda.Stream(priority=0)
    v_args, v_grid = F.stencil_args(v_out, v_in), F.stencil_grid(n_st)
    n_v = v_grid[0] * v_grid[1]

    def w_args(n):
        elems = n * cps_w * 256
        return F.saxpy_f32_args(wy[:elems], wx[:elems], 0.5), F.saxpy_grid(elems)

    def alone(k, grid, a):
        flush.zero_()
        torch.cuda.synchronize()
        h = rt.launch(k, grid, a, stream=A)
        rt.sync(h)
        t0, t1 = _span(rt.events(h, 1))
        return (t1 - t0) / 1e3

    for _ in range(2):
        alone(k_v, v_grid, v_args)
    t_v = float(np.median([alone(k_v, v_grid, v_args) for _ in range(5)]))
    rng = gen.rng(2000 + rank)
    check_rows = sorted(set(int(r) for r in gen.rng(2050 + rank).integers(1, n_st - 1, 6)))
    slabs = {r: v_in[r - 1:r + 2].cpu().numpy() for r in check_rows}
    import bench_check as BC

    def victim_rows_err():
        """Sampled output rows of the last victim run against NumPy fp64 (3-row slabs)."""
        worst = 0.0
        for r in check_rows:
            ref, den = BC.stencil5_f32(slabs[r])
            got = v_out[r].cpu().numpy()
            d = np.maximum(np.abs(ref[1]), den[1])
            worst = max(worst, float(np.max(np.abs(got - ref[1]) / np.where(d > 0, d, 1))))
        return worst
    rows = []
    with ClockSampler(physical_gpu_index(local)) as clk:
        for n in widths:
            wa, wg = w_args(n)
            t_w = float(np.median([alone(k_w, wg, wa) for _ in range(5)]))
            lat, start, tflep, tflep_r, viol, ok = [], [], [], [], 0, 0
            for trial in range(2 * (args.warmup + args.steps)):
                refill = trial % 2 == 1 and n < rt.num_sms
                tstar = int(rng.integers(n_v // 4, n_v // 2))
                flush.zero_()
                torch.cuda.synchronize()
                rt.arm_next_trigger(tstar, n)
                h_v = rt.launch(k_v, v_grid, v_args, priority=0, stream=A)
                h_w = rt.launch(k_w, wg, wa, priority=1, stream=B)
                if refill:
                    # f1: once the waiting kernel is done, re-spread the victim over all SMs
                    rt.sync(h_w, timeout_ns=10_000_000_000)
                    try:
                        rt.preempt(h_v, n)          # host view of the device-triggered request
                        rt.refill(h_v)
                    except F.FlepError:
                        pass                        # the victim already finished
                rt.wait_epoch(h_v, timeout_ns=10_000_000_000)
                if rt.query(h_v).state == F.STATE_PREEMPTED:
                    rt.sync(h_w, timeout_ns=10_000_000_000)
                    rt.resume(h_v)
                rt.sync(h_v, timeout_ns=10_000_000_000)
                rt.sync(h_w, timeout_ns=10_000_000_000)
                info = rt.query(h_v)
                ep = rt.epoch_info(h_v, 1)
                ev1 = rt.events(h_v, 1)
                evs = list(ev1)
                for e_ in range(2, info.epoch + 1):
                    evs += list(rt.events(h_v, e_))
                evw = rt.events(h_w, 1)
                if trial < 2 * args.warmup or ep.t_trigger == 0:
                    continue
                if refill:
                    v0, v1 = _span(evs)
                    w0, w1 = _span(evw)
                    tflep_r.append((max(v1, w1) - v0) / 1e3)
                    continue
                yielded = [e for e in ev1 if e.reason == F.REASON_YIELD]
                if n < rt.num_sms:
                    viol += sum(1 for e in ev1 if (e.reason == F.REASON_YIELD) != (e.smid < n))
                v0, v1 = _span(evs)
                w0, w1 = _span(evw)
                if yielded:
                    lat.append((max(e.t_exit for e in yielded) - ep.t_trigger) / 1e3)
                start.append((w0 - ep.t_trigger) / 1e3)
                tflep.append((max(v1, w1) - v0) / 1e3)
                ok += 1
            t_org = t_v + t_w
            verr = victim_rows_err()
            rows.append({"n_sms": n, "trials": ok, "victim_rows_max_rel": verr, "victim_parity_ok": bool(verr <= 1e-5), "yield_latency_us_p50": round(float(np.median(lat)), 3) if lat else None,
                         "yield_latency_us_max": round(float(np.max(lat)), 3) if lat else None,
                         "waiting_start_us_p50": round(float(np.median(start)), 3),
                         "t_flep_us": round(float(np.median(tflep)), 2), "t_org_us": round(t_org, 2),
                         "t_victim_alone_us": round(t_v, 2), "t_waiting_alone_us": round(t_w, 2),
                         "overhead": round((float(np.median(tflep)) - t_org) / t_org, 4),
                         "t_flep_refill_us": round(float(np.median(tflep_r)), 2) if tflep_r else None,
                         "overhead_with_refill": (round((float(np.median(tflep_r)) - t_org) / t_org, 4)
                                                  if tflep_r else None),
                         "I3_violations": viol})
    clocks = clk.summary()
    temporal = rows[-1]
    for r in rows:
        r["overhead_reduction_vs_temporal"] = (round(1.0 - r["overhead"] / temporal["overhead"], 4)
                                               if temporal["overhead"] > 0 else None)
        r["overhead_reduction_vs_temporal_with_refill"] = (
            round(1.0 - r["overhead_with_refill"] / temporal["overhead"], 4)
            if r.get("overhead_with_refill") is not None and temporal["overhead"] > 0 else None)
        r["latency_vs_temporal"] = (round(r["yield_latency_us_p50"] / temporal["yield_latency_us_p50"], 3)
                                    if r["yield_latency_us_p50"] and temporal["yield_latency_us_p50"] else None)
    rt.close()
    out = {"metric": METRIC, "value": rows[0]["overhead_reduction_vs_temporal_with_refill"],
           "unit": "fraction (1 - ovh_spatial / ovh_temporal)",
           "value_definition": "preemption-overhead reduction of an 8-SM spatial yield (with refill) vs a full-GPU "
                               "yield, overhead = (T_FLEP - T_org) / T_org (P:297, Fig. 15)",
           "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "higher_is_better": True,
           "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic (seeded)",
           "config": {"workload": "configs[2]: spatial preemption of stencil5 fp32 16384^2 (victim) by SAXPY-f32 "
                                  "with n*k_wait blocks (waiting kernel) for n in {8,16,32,74} and 148 (temporal)",
                      "victim_chunk": 1, "poll": 1, "l2": "flushed between trials"},
           "per_width": rows,
           "victim_parity_ok": all(r["victim_parity_ok"] for r in rows),
           "spatial_cheaper_than_full": all((r["overhead_with_refill"] if r["overhead_with_refill"] is not None
                                             else 1e9) < temporal["overhead"] for r in rows[:-1]),
           "spatial_yield_latency_lower_than_full": all(
               (r["yield_latency_us_p50"] or 1e9) < (temporal["yield_latency_us_p50"] or 0) for r in rows[:-1]),
           "clocks": clocks}
    _emit(out, rank, args)
    barrier(world)
    return out


def _rank_tables(num_sms, die):
    """Yield orders (rank[smid]; a spatial request for n releases the SMs with rank < n):
    ascending smid (the paper's ID < spa_P), die-packed (one die's SMs first) and die-balanced
    (the dies alternate), from a measured smid -> die map (probes/probe7.cu)."""
    tables = {"ascending": list(range(num_sms))}
    if die is None or len(die) < num_sms:
        return tables
    d0 = [s for s in range(num_sms) if die[s] == 0]
    d1 = [s for s in range(num_sms) if die[s] == 1]
    packed = d0 + d1
    balanced = [x for pair in zip(d0, d1) for x in pair] + d0[len(d1):] + d1[len(d0):]
    for name, order in (("die_packed", packed), ("die_balanced", balanced)):
        r = [0] * num_sms
        for k, smid in enumerate(order):
            r[smid] = k
        tables[name] = r
    return tables


def run_spatial_f1(args, rank, world, local):
    """SURVEY f1 beyond refill (Fig. 16): a 16384^2 stencil victim (counter worker,
    C = K = 1) yields n SMs to a SAXPY-f32 waiting kernel.
    (A) "More than enough SMs": the waiting kernel is sized for n_need = 8 SMs (8 x k_wait CTAs)
        and the request yields n = 8, 12, 16, 24, 32: waiting-kernel turnaround (request -> its
        last CTA), co-run time T_FLEP and its overhead over T_org.
    (B) Which SMs: rank tables ascending smid (paper), die-packed and die-balanced (measured
        smid -> die map, FLEP_DIE_MAP or profiles/r01_sm_die_map.json) at n = 16, 32, 74 with the
        waiting kernel sized for n SMs: yield latency, waiting turnaround, overhead; I3 checked
        against each table."""
    import os
    import torch
    from bench import ClockSampler, L2Flush, barrier, physical_gpu_index, ROOT
    from paper_conf_asplos_wulzj17_b200 import flep as F
    torch.cuda.set_device(local)
    rt = F.Runtime(device=local, exec_on_user_stream=True)
    die_path = os.environ.get("FLEP_DIE_MAP") or os.path.join(ROOT, "profiles", "r01_sm_die_map.json")
    try:
        with open(die_path) as fh:
            die = json.load(fh)["die"]
    except Exception:
        die = None
    n_st = 16384
    g = torch.Generator(device="cuda")
    g.manual_seed(4 + rank)
    v_in = torch.rand(n_st, n_st, device="cuda", generator=g)
    v_out = torch.empty_like(v_in)
    k_v = rt.register_kernel(F.BODY_STENCIL5_F32, chunk=1, poll=1, name="victim")
    k_w = rt.register_kernel(F.BODY_SAXPY_F32, chunk=1, poll=1, name="waiting")
    cps_w, _ = rt.workers_for(F.BODY_SAXPY_F32)
    n_max = 74 * cps_w * 256
    wx = torch.rand(n_max, device="cuda", generator=g)
    wy = torch.rand(n_max, device="cuda", generator=g)
    flush = L2Flush(torch)
    A = torch.cuda.Stream(priority=-2)
    B = torch.cuda.Stream(priority=0)
    v_args, v_grid = F.stencil_args(v_out, v_in), F.stencil_grid(n_st)
    n_v = v_grid[0] * v_grid[1]
    rng = gen.rng(3000 + rank)

    def w_args(n):
        elems = n * cps_w * 256
        return F.saxpy_f32_args(wy[:elems], wx[:elems], 0.5), F.saxpy_grid(elems)

    def alone(k, grid, a):
        flush.zero_()
        torch.cuda.synchronize()
        h = rt.launch(k, grid, a, stream=A)
        rt.sync(h)
        t0, t1 = _span(rt.events(h, 1))
        return (t1 - t0) / 1e3

    def trials(n, wa, wg, table, reps):
        lat, wturn, tflep, viol = [], [], [], 0
        for trial in range(reps + 2):
            tstar = int(rng.integers(n_v // 4, n_v // 2))
            flush.zero_()
            torch.cuda.synchronize()
            rt.arm_next_trigger(tstar, n)
            h_v = rt.launch(k_v, v_grid, v_args, priority=0, stream=A)
            h_w = rt.launch(k_w, wg, wa, priority=1, stream=B)
            rt.wait_epoch(h_v, timeout_ns=10_000_000_000)
            if rt.query(h_v).state == F.STATE_PREEMPTED:
                rt.sync(h_w, timeout_ns=10_000_000_000)
                rt.resume(h_v)
            rt.sync(h_v, timeout_ns=10_000_000_000)
            rt.sync(h_w, timeout_ns=10_000_000_000)
            info = rt.query(h_v)
            ep = rt.epoch_info(h_v, 1)
            ev1 = rt.events(h_v, 1)
            evs = list(ev1)
            for e_ in range(2, info.epoch + 1):
                evs += list(rt.events(h_v, e_))
            evw = rt.events(h_w, 1)
            if trial < 2 or ep.t_trigger == 0:
                continue
            viol += sum(1 for e in ev1 if (e.reason == F.REASON_YIELD) != (table[e.smid] < n))
            y = [e.t_exit for e in ev1 if e.reason == F.REASON_YIELD]
            if y:
                lat.append((max(y) - ep.t_trigger) / 1e3)
            v0, v1 = _span(evs)
            w0, w1 = _span(evw)
            wturn.append((w1 - ep.t_trigger) / 1e3)
            tflep.append((max(v1, w1) - v0) / 1e3)
        med = lambda v: round(float(np.median(v)), 3) if v else None  # noqa: E731
        return {"yield_latency_us_p50": med(lat), "waiting_turnaround_us_p50": med(wturn),
                "t_flep_us": med(tflep), "I3_violations": viol, "trials": len(tflep)}

    for _ in range(2):
        alone(k_v, v_grid, v_args)
    t_v = float(np.median([alone(k_v, v_grid, v_args) for _ in range(5)]))
    reps = max(10, args.steps // 4)
    more, which = [], []
    tables = _rank_tables(rt.num_sms, die)
    with ClockSampler(physical_gpu_index(local)) as clk:
        rt.set_rank_table(tables["ascending"])
        wa, wg = w_args(8)
        t_w8 = float(np.median([alone(k_w, wg, wa) for _ in range(5)]))
        for n in (8, 12, 16, 24, 32):
            r = trials(n, wa, wg, tables["ascending"], reps)
            t_org = t_v + t_w8
            r.update({"n_need": 8, "n_sms": n, "t_org_us": round(t_org, 2), "t_waiting_alone_us": round(t_w8, 2),
                      "overhead": round((r["t_flep_us"] - t_org) / t_org, 4) if r["t_flep_us"] else None})
            more.append(r)
        for name, table in tables.items():
            rt.set_rank_table(table)
            for n in (16, 32, 74):
                wa, wg = w_args(n)
                t_w = float(np.median([alone(k_w, wg, wa) for _ in range(3)]))
                r = trials(n, wa, wg, table, reps)
                t_org = t_v + t_w
                r.update({"table": name, "n_sms": n, "t_org_us": round(t_org, 2),
                          "overhead": round((r["t_flep_us"] - t_org) / t_org, 4) if r["t_flep_us"] else None})
                which.append(r)
        rt.set_rank_table(tables["ascending"])
    rt.close()
    base = more[0]["waiting_turnaround_us_p50"]
    for r in more:
        r["waiting_speedup_vs_n_need"] = round(base / r["waiting_turnaround_us_p50"], 3) \
            if base and r["waiting_turnaround_us_p50"] else None
    best = max((r["waiting_speedup_vs_n_need"] or 0) for r in more)
    out = {"metric": METRIC, "value": best, "unit": "x",
           "value_definition": "largest waiting-kernel turnaround speedup from yielding more SMs than its grid "
                               "needs (n_need = 8), P:383 Fig. 16",
           "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "higher_is_better": True,
           "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic (seeded)",
           "config": {"workload": "stencil5 fp32 16384^2 victim (C=K=1) spatially preempted by SAXPY-f32",
                      "die_map": die_path if die else None, "trials_per_point": reps,
                      "l2": "flushed between trials"},
           "more_than_enough": more, "rank_tables": which, "clocks": clk.summary()}
    _emit(out, rank, args)
    barrier(world)
    return out


# ------------------------------------------------------------------------------------------
def run_corun1(args, rank, world, local):
    """configs[0]: LP SAXPY-int32 2^20 preempted mid-run by HP SAXPY-int32 2^16 (device trigger,
    temporal); exactly-once coverage and bit-exact results checked against a NumPy reference (bench_check) every step."""
    import torch
    import bench_check as W
    from bench import ClockSampler, L2Flush, barrier, physical_gpu_index
    from paper_conf_asplos_wulzj17_b200 import flep as F
    torch.cuda.set_device(local)
    rt = F.Runtime(device=local, exec_on_user_stream=True, coverage=True)
    T = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()  # noqa: E731
    n_lp, n_hp, a_lp, a_hp = 1 << 20, 1 << 16, 1664525, 22695477
    x, y = gen.saxpy_i32_inputs(n_lp, seed=1)
    x2, y2 = gen.saxpy_i32_inputs(n_hp, seed=11)
    ref_lp, ref_hp = W.saxpy_i32(a_lp, x, y), W.saxpy_i32(a_hp, x2, y2)
    xd, y0, yd = T(x), T(y), T(y)
    x2d, y20, y2d = T(x2), T(y2), T(y2)
    k_lp = rt.register_kernel(F.BODY_SAXPY_I32, chunk=1, poll=1, ctas_per_sm=args.corun_cps)
    k_hp = rt.register_kernel(F.BODY_SAXPY_I32, chunk=1, poll=1)
    flush = L2Flush(torch)
    A = torch.cuda.Stream(priority=-2)
    B = torch.cuda.Stream(priority=0)
    nb = n_lp // 256
    rng = gen.rng(3000 + rank)
    lat, drain, hpt, bad, pre, hpt_fifo = [], [], [], 0, 0, []
    with ClockSampler(physical_gpu_index(local)) as clk:
        # FIFO reference (no preemption): the same arrival point is only stamped (trigger width 0),
        # the HP kernel waits behind the persistent LP workers
        for i in range(args.warmup + args.steps):
            yd.copy_(y0)
            y2d.copy_(y20)
            flush.zero_()
            torch.cuda.synchronize()
            tstar = int(rng.integers(nb // 4, 3 * nb // 4))
            rt.arm_next_trigger(tstar, 0)
            h = rt.launch(k_lp, F.saxpy_grid(n_lp), F.saxpy_i32_args(yd, xd, a_lp), priority=0, stream=A)
            h2 = rt.launch(k_hp, F.saxpy_grid(n_hp), F.saxpy_i32_args(y2d, x2d, a_hp), priority=1, stream=B)
            rt.sync(h, timeout_ns=10_000_000_000)
            rt.sync(h2, timeout_ns=10_000_000_000)
            ep = rt.epoch_info(h, 1)
            if i >= args.warmup and ep.t_trigger:
                hpt_fifo.append((_span(rt.events(h2, 1))[1] - ep.t_trigger) / 1e3)
        rng = gen.rng(3000 + rank)
        for i in range(args.warmup + args.steps):
            yd.copy_(y0)
            y2d.copy_(y20)
            flush.zero_()
            torch.cuda.synchronize()
            tstar = int(rng.integers(nb // 4, 3 * nb // 4))
            rt.arm_next_trigger(tstar, rt.num_sms)
            h = rt.launch(k_lp, F.saxpy_grid(n_lp), F.saxpy_i32_args(yd, xd, a_lp), priority=0, stream=A)
            h2 = rt.launch(k_hp, F.saxpy_grid(n_hp), F.saxpy_i32_args(y2d, x2d, a_hp), priority=1, stream=B)
            rt.wait_epoch(h, timeout_ns=10_000_000_000)
            preempted = rt.query(h).state == F.STATE_PREEMPTED
            rt.sync(h2, timeout_ns=10_000_000_000)
            if preempted:
                rt.resume(h)
            rt.sync(h, timeout_ns=10_000_000_000)
            ep = rt.epoch_info(h, 1)
            ev_hp = rt.events(h2, 1)
            ok = (np.all(rt.coverage_np(h, nb) == 1) and np.array_equal(yd.cpu().numpy(), ref_lp)
                  and np.array_equal(y2d.cpu().numpy(), ref_hp))
            if i < args.warmup:
                continue
            bad += 0 if ok else 1
            if preempted and ep.t_trigger:
                pre += 1
                hs, he = _span(ev_hp)
                lat.append((hs - ep.t_trigger) / 1e3)
                drain.append((ep.t_end - ep.t_trigger) / 1e3)
                hpt.append((he - ep.t_trigger) / 1e3)
    rt.close()
    out = {"metric": METRIC, "value": round(float(np.median(drain)), 3) if drain else None, "unit": "us",
           "value_definition": "full-GPU preemption latency: device request -> last LP CTA gone, p50",
           "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "higher_is_better": False,
           "scaling": "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic (seeded)",
           "config": {"workload": "configs[0]: LP SAXPY-int32 2^20 preempted by HP SAXPY-int32 2^16",
                      "lp_ctas_per_sm": args.corun_cps, "chunk": 1, "poll": 1},
           "preempted_steps": pre, "wrong_results": bad,
           "waiting_start_us_p50": round(float(np.median(lat)), 3) if lat else None,
           "hp_turnaround_us_p50": round(float(np.median(hpt)), 3) if hpt else None,
           "hp_turnaround_fifo_us_p50": round(float(np.median(hpt_fifo)), 3) if hpt_fifo else None,
           "hp_speedup_vs_fifo": (round(float(np.median(hpt_fifo)) / float(np.median(hpt)), 2)
                                  if hpt and hpt_fifo else None),
           "drain_us_max": round(float(np.max(drain)), 3) if drain else None,
           "clocks": clk.summary()}
    _emit(out, rank, args)
    barrier(world)
    return out


# ------------------------------------------------------------------------------------------
def run_gemm_preempt(args, rank, world, local):
    """Full-GPU preemption of the dense contraction: LP bf16 GEMM 8192^3 (C = A B^T, tcgen05)
    preempted at a random tile by HP stencil5 4096^2 (device self-trigger, temporal), then
    resumed. Latency = request -> last GEMM CTA gone (device %globaltimer). Each step's result
    must be bit-identical to an uninterrupted run of the same binary (SURVEY §8(c) parity), and a
    sample of C is checked against fp64 dot products (bench_check, 2e-2 relative)."""
    import torch
    import bench_check as W
    from bench import ClockSampler, L2Flush, barrier, physical_gpu_index
    from paper_conf_asplos_wulzj17_b200 import flep as F
    torch.cuda.set_device(local)
    rt = F.Runtime(device=local, exec_on_user_stream=True)
    M = N = K = 8192
    g = torch.Generator(device="cuda")
    g.manual_seed(8 + rank)
    A_ = (torch.rand(M, K, device="cuda", generator=g) * 2 - 1).to(torch.bfloat16)
    B_ = (torch.rand(N, K, device="cuda", generator=g) * 2 - 1).to(torch.bfloat16)
    C_ = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    st_in = torch.rand(4096, 4096, device="cuda", generator=g)
    st_out = torch.empty_like(st_in)
    in_tile = bool(args.gemm_in_tile)
    pair = int(getattr(args, "gemm_pair", 0))             # 1: the CTA-pair body (R32), 2: its wide tile
    body = {0: F.BODY_GEMM_BF16, 1: F.BODY_GEMM_BF16_2SM, 2: F.BODY_GEMM_BF16_2SM_W}[pair]
    k_lp = rt.register_kernel(body, chunk=1, poll=1, name="gemm", in_tile=in_tile)
    k_hp = rt.register_kernel(F.BODY_STENCIL5_F32, chunk=2, poll=1, prefetch=True, name="stencil")
    lp_args = F.gemm_args(C_, A_, B_)
    lp_grid = {0: F.gemm_grid, 1: F.gemm2_grid, 2: F.gemm2w_grid}[pair](M, N)
    hp_args, hp_grid = F.stencil_args(st_out, st_in), F.stencil_grid(4096)
    nb = lp_grid[0] * lp_grid[1]
    flush = L2Flush(torch)
    SA = torch.cuda.Stream(priority=-2)
    SB = torch.cuda.Stream(priority=0)
    # uninterrupted reference of the same binary
    h = rt.launch(k_lp, lp_grid, lp_args, stream=SA)
    rt.sync(h)
    torch.cuda.synchronize()
    C_ref = C_.clone()
    rng = gen.rng(5000 + rank)
    lat, drain, hpt, bad, pre, epochs, early = [], [], [], 0, 0, [], 0
    with ClockSampler(physical_gpu_index(local)) as clk:
        for i in range(args.warmup + args.steps):
            C_.zero_()
            flush.zero_()
            torch.cuda.synchronize()
            tstar = int(rng.integers(nb // 4, 3 * nb // 4))
            rt.arm_next_trigger(tstar, rt.num_sms)
            h = rt.launch(k_lp, lp_grid, lp_args, priority=0, stream=SA)
            h2 = rt.launch(k_hp, hp_grid, hp_args, priority=1, stream=SB)
            rt.wait_epoch(h, timeout_ns=20_000_000_000)
            preempted = rt.query(h).state == F.STATE_PREEMPTED
            rt.sync(h2, timeout_ns=20_000_000_000)
            if preempted:
                rt.resume(h)
            rt.sync(h, timeout_ns=20_000_000_000)
            torch.cuda.synchronize()
            ep = rt.epoch_info(h, 1)
            ev_hp = rt.events(h2, 1)
            same = bool(torch.equal(C_, C_ref))
            if i < args.warmup:
                continue
            bad += 0 if same else 1
            if preempted and ep.t_trigger:
                pre += 1
                hs, he = _span(ev_hp)
                if hs < ep.t_trigger:
                    early += 1         # the HP's CTAs fit beside the GEMM worker (1 CTA/SM)
                else:
                    lat.append((hs - ep.t_trigger) / 1e3)
                drain.append((ep.t_end - ep.t_trigger) / 1e3)
                hpt.append((he - ep.t_trigger) / 1e3)
                epochs.append(rt.query(h).epoch)
    # spot check of the last result (rows x cols sampled; fp64 dot products of bf16 values)
    r_idx = gen.rng(9).integers(0, M, 16)
    c_idx = gen.rng(10).integers(0, N, 64)
    a = A_[r_idx].view(torch.int16).cpu().numpy().view(np.uint16)
    b = B_[c_idx].view(torch.int16).cpu().numpy().view(np.uint16)
    ref = W.gemm_bf16(a, b)
    got = C_[r_idx][:, c_idx].float().cpu().numpy()
    rms = float(np.sqrt(np.mean(ref ** 2)))
    worst = float(np.max(np.abs(got - ref) / (np.abs(ref) + rms)))
    rt.close()
    out = {"metric": METRIC, "value": round(float(np.median(drain)), 3) if drain else None, "unit": "us",
           "value_definition": "full-GPU preemption latency of a bf16 GEMM 8192^3 victim: device request -> "
                               "last GEMM CTA gone, p50",
           "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "higher_is_better": False,
           "scaling": "weak", "vs_baseline": None, "dtype": "bf16", "data": "synthetic (seeded)",
           "config": {"workload": {0: "LP GEMM bf16 8192^3 (tcgen05, 128x256 tiles)",
                                   1: "LP GEMM bf16 8192^3 (tcgen05 cta_group::2, 256x256 tiles on CTA pairs)",
                                   2: "LP GEMM bf16 8192^3 (tcgen05 cta_group::2, 256x512 tiles on CTA pairs)"}[pair]
                                  + " preempted by HP stencil5 4096^2",
                      "chunk": 1, "poll": 1, "in_tile": in_tile, "pair": pair},
           "preempted_steps": pre, "not_bit_identical_to_uninterrupted": bad,
           "sample_max_rel": worst, "tol": 2e-2,
           "drain_us": {"p50": round(float(np.median(drain)), 3) if drain else None,
                        "p99": round(float(np.percentile(drain, 99)), 3) if drain else None,
                        "max": round(float(np.max(drain)), 3) if drain else None},
           "waiting_start_us_p50": round(float(np.median(lat)), 3) if lat else None,
           "hp_started_before_request": early,
           "note": "the HP stencil's CTAs (no smem) can be resident beside the GEMM worker (1 CTA/SM, "
                   "~197 KB smem), so it often starts before the request; drain_us is the GEMM's yield",
           "clocks": clk.summary()}
    _emit(out, rank, args)
    barrier(world)
    return out


def run_clc(args, rank, world, local):
    """CLC task fetch vs the atomic counter (R25) on configs[1] kernels.

    (1) Co-run: LP SpMV-CSR 2^20 rows on a low-priority stream; the HP stencil5 4096^2 is released
        by the host ~20 us after the LP launch on a high-priority stream. Variants: CLC victim with
        no request (the hardware's queue yields: try_cancel fails while a higher-priority grid is
        pending), counter victim with the FLEP request issued by the host at the HP's release
        (flep_preempt, then resume after the HP), counter victim without a request (the HP waits
        for the whole LP). Per step (device %globaltimer): HP turnaround = HP last CTA exit - LP
        first CTA entry, and LP span. Spot parity of the last LP result (bench_check).
    (2) Wrapper overhead of both fetch variants against the unwrapped kernels (dithered CUDA
        events, L2 flushed)."""
    import torch
    from bench import (ClockSampler, L2Flush, Workload, barrier, physical_gpu_index, spot_parity,
                       STENCIL_N, SPMV_ROWS)
    from paper_conf_asplos_wulzj17_b200 import flep as F
    from paper_conf_asplos_wulzj17_b200.calibrate import dither, event_mean_us
    torch.cuda.set_device(local)
    rt = F.Runtime(device=local, exec_on_user_stream=True)
    wl = Workload(torch)
    flush = L2Flush(torch)
    lo, hi = torch.cuda.Stream(priority=0), torch.cuda.Stream(priority=-2)
    lp_args = F.spmv_args(wl.d_y, wl.d_rowptr, wl.d_col, wl.d_val, wl.d_x)
    hp_args = F.stencil_args(wl.d_out, wl.d_in)
    lp_grid, hp_grid = F.spmv_grid(SPMV_ROWS), F.stencil_grid(STENCIL_N)
    k_clc = rt.register_kernel(F.BODY_SPMV_CSR_F32, chunk=1, poll=1, clc=True, name="spmv_clc")
    k_ctr = rt.register_kernel(F.BODY_SPMV_CSR_F32, chunk=1, poll=1, name="spmv")
    k_hp = rt.register_kernel(F.BODY_STENCIL5_F32, chunk=4, poll=1, name="stencil")
    variants = [("clc_no_request", k_clc, False), ("clc_flep_request", k_clc, True),
                ("counter_flep_request", k_ctr, True), ("counter_no_request", k_ctr, False)]
    res = {v[0]: {"hp_turnaround": [], "lp_span": [], "yields": [], "lp_after_hp": [], "hp_start": []}
           for v in variants}

    def spin_us(us):
        t0 = time.perf_counter()
        while time.perf_counter() - t0 < us * 1e-6:
            pass
    with ClockSampler(physical_gpu_index(local)) as clk:
        for i in range(args.warmup + args.steps):
            for name, k_lp, request in variants:
                with torch.cuda.stream(lo):
                    flush.zero_()
                torch.cuda.synchronize()
                h = rt.launch(k_lp, lp_grid, lp_args, priority=0, stream=lo)
                spin_us(20)
                if request:
                    rt.preempt(h, rt.num_sms)
                h2 = rt.launch(k_hp, hp_grid, hp_args, priority=1, stream=hi)
                rt.sync(h2, timeout_ns=10_000_000_000)
                if request and name.startswith("clc"):
                    # a CLC request is in force at once; resume withdraws it (the preempted grid
                    # may have completed meanwhile: its queued CTAs still start, R25)
                    try:
                        rt.resume(h)
                    except F.FlepError:
                        assert rt.query(h).state == F.STATE_DONE
                elif request:
                    rt.wait_epoch(h, timeout_ns=10_000_000_000)
                    if rt.query(h).state == F.STATE_PREEMPTED:
                        rt.resume(h)
                rt.sync(h, timeout_ns=10_000_000_000)
                torch.cuda.synchronize()
                if i < args.warmup:
                    continue
                lp_ev = rt.events(h, 1)
                gen_now = max(e.epoch for e in lp_ev)    # stale slots of cancelled CTAs keep older gens
                lp_ev = [e for e in lp_ev if e.epoch == gen_now]
                lp0 = min(e.t_entry for e in lp_ev)
                hp_ev = rt.events(h2, 1)
                hp1 = max(e.t_exit for e in hp_ev)
                hp0 = min(e.t_entry for e in hp_ev)
                q = rt.query(h)
                lp_end = max(max(e.t_exit for e in lp_ev),
                             max((e.t_exit for e in rt.events(h, q.epoch)), default=0))
                r = res[name]
                r["hp_turnaround"].append((hp1 - lp0) / 1e3)
                r["lp_span"].append((lp_end - lp0) / 1e3)
                r["yields"].append(sum(1 for e in lp_ev if e.reason == F.REASON_YIELD))
                # victim CTAs that started after the waiting kernel's first CTA (refills of freed
                # slots by the victim's own pending CTAs) and the HP's start after the LP's
                r["lp_after_hp"].append(sum(1 for e in lp_ev if e.t_entry > hp0))
                r["hp_start"].append((hp0 - lp0) / 1e3)
    parity = spot_parity(wl, torch)
    reps = max(args.reps, 20)

    def timed(fn):
        ts = []
        for r in range(reps + 2):
            with torch.cuda.stream(lo):
                flush.zero_()
                dither(torch)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(lo)
            h = fn()
            e1.record(lo)
            e1.synchronize()
            if h is not None:
                rt.sync(h)
            if r >= 2:
                ts.append(e0.elapsed_time(e1) * 1e3)
        return round(event_mean_us(ts), 3)
    over = {}
    n_sx = 1 << 20
    xs = torch.randint(-2 ** 31, 2 ** 31 - 1, (n_sx,), dtype=torch.int32, device="cuda")
    ys = torch.randint(-2 ** 31, 2 ** 31 - 1, (n_sx,), dtype=torch.int32, device="cuda")
    cases = [("spmv", F.BODY_SPMV_CSR_F32, lp_grid, lp_args, dict(chunk=2, poll=2), dict(chunk=2, poll=2)),
             ("spmv_c1k1", F.BODY_SPMV_CSR_F32, lp_grid, lp_args, dict(chunk=1, poll=1), dict(chunk=1, poll=1)),
             ("stencil", F.BODY_STENCIL5_F32, hp_grid, hp_args, dict(chunk=4, poll=1), dict(chunk=1, poll=4)),
             ("saxpy_i32_2^20", F.BODY_SAXPY_I32, F.saxpy_grid(n_sx), F.saxpy_i32_args(ys, xs, 3),
              dict(chunk=16, poll=2, prefetch=True, async_poll=True), dict(chunk=8, poll=2))]
    for name, body, grid, a, ckw, clkw in cases:
        k_c = rt.register_kernel(body, clc=True, **clkw)
        k_a = rt.register_kernel(body, **ckw)
        t_u = timed(lambda: rt.launch_unwrapped(body, grid, a, stream=lo))
        t_c = timed(lambda: rt.launch(k_c, grid, a, stream=lo))
        t_a = timed(lambda: rt.launch(k_a, grid, a, stream=lo))
        over[name] = {"unwrapped_us": t_u, "clc_us": t_c, "counter_us": t_a, "clc_config": clkw,
                      "counter_config": ckw, "clc_overhead_pct": round((t_c / t_u - 1) * 100, 2),
                      "counter_overhead_pct": round((t_a / t_u - 1) * 100, 2)}
    rt.close()

    def q(v, p):
        return round(float(np.percentile(v, p)), 3) if v else None
    summ = {k: {"hp_turnaround_us": {"p50": q(r["hp_turnaround"], 50), "p99": q(r["hp_turnaround"], 99)},
                "lp_span_us": {"p50": q(r["lp_span"], 50)},
                "first_wave_yield_exits_p50": q(r["yields"], 50),
                "hp_first_cta_us_p50": q(r["hp_start"], 50),
                "lp_ctas_started_after_hp_p50": q(r["lp_after_hp"], 50)} for k, r in res.items()}
    out = {"metric": METRIC, "value": summ["clc_no_request"]["hp_turnaround_us"]["p50"], "unit": "us",
           "value_definition": "HP turnaround (HP last CTA exit - LP first CTA entry, device %globaltimer) with a CLC "
                               "victim and no preemption request, p50; the HP is released ~20 us after the LP",
           "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "higher_is_better": False,
           "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic (seeded; synth/gen.py)",
           "config": {"workload": "configs[1] kernels: LP SpMV-CSR 2^20 rows (low-priority stream) and HP stencil5 "
                                  "4096^2 (high-priority stream, host-released ~20 us after the LP)",
                      "l2": "flushed before every step"},
           "variants": summ, "wrapper_overhead": over, "parity": parity, "clocks": clk.summary()}
    _emit(out, rank, args)
    barrier(world)
    return out


def run_delay(args, rank, world, local):
    """Delay sweep (Fig. 9): the HP kernel (stencil5 4096^2) arrives when the
    LP victim (SpMV-CSR 2^20 rows, counter worker C = K = 1) has handed out a fraction d of its
    blocks (device self-trigger at block d*N), d = 0.1 .. 0.9. FLEP: the trigger is a temporal
    request; FIFO: the same trigger only stamps the arrival (n = 0), the HP waits for the LP.
    HP turnaround = HP last CTA exit - arrival (device %globaltimer); speedup = FIFO / FLEP, next
    to the zero-overhead bound (T_LP (1 - d) + T_HP) / T_HP from the standalone times."""
    import torch
    from bench import (ClockSampler, L2Flush, Workload, barrier, physical_gpu_index, spot_parity,
                       STENCIL_N, SPMV_ROWS)
    from paper_conf_asplos_wulzj17_b200 import flep as F
    torch.cuda.set_device(local)
    rt = F.Runtime(device=local, exec_on_user_stream=True)
    wl = Workload(torch)
    flush = L2Flush(torch)
    A, B = torch.cuda.Stream(priority=-2), torch.cuda.Stream(priority=0)
    lp_args = F.spmv_args(wl.d_y, wl.d_rowptr, wl.d_col, wl.d_val, wl.d_x)
    hp_args = F.stencil_args(wl.d_out, wl.d_in)
    lp_grid, hp_grid = F.spmv_grid(SPMV_ROWS), F.stencil_grid(STENCIL_N)
    n_lp = lp_grid[0]
    k_lp = rt.register_kernel(F.BODY_SPMV_CSR_F32, chunk=1, poll=1, name="spmv")
    k_hp = rt.register_kernel(F.BODY_STENCIL5_F32, chunk=1, poll=4, clc=True, name="stencil")

    def alone(k, grid, a):
        ts = []
        for _ in range(12):
            flush.zero_()
            torch.cuda.synchronize()
            h = rt.launch(k, grid, a, stream=A)
            rt.sync(h)
            ev = rt.events(h, 1)
            ts.append((max(e.t_exit for e in ev) - min(e.t_entry for e in ev)) / 1e3)
        return float(np.median(ts[2:]))
    t_lp, t_hp = alone(k_lp, lp_grid, lp_args), alone(k_hp, hp_grid, hp_args)
    reps = max(4, args.steps // 10)
    points = []
    with ClockSampler(physical_gpu_index(local)) as clk:
        for d in [i / 10 for i in range(1, 10)]:
            res = {}
            for mode in ("fifo", "flep"):
                tt = []
                for r in range(reps + 1):
                    with torch.cuda.stream(A):
                        flush.zero_()
                        e0 = torch.cuda.Event()
                        e0.record(A)
                    rt.arm_next_trigger(int(d * n_lp), rt.num_sms if mode == "flep" else 0)
                    h = rt.launch(k_lp, lp_grid, lp_args, priority=0, stream=A)
                    B.wait_event(e0)
                    h2 = rt.launch(k_hp, hp_grid, hp_args, priority=1, stream=B)
                    rt.wait_epoch(h, timeout_ns=10_000_000_000)
                    pre = rt.query(h).state == F.STATE_PREEMPTED
                    rt.sync(h2, timeout_ns=10_000_000_000)
                    if pre:
                        rt.resume(h)
                    rt.sync(h, timeout_ns=10_000_000_000)
                    torch.cuda.synchronize()
                    ep = rt.epoch_info(h, 1)
                    hp_end = max(e.t_exit for e in rt.events(h2, 1))
                    if r >= 1 and ep.t_trigger:
                        tt.append((hp_end - ep.t_trigger) / 1e3)
                res[mode] = float(np.median(tt)) if tt else None
            bound = (t_lp * (1 - d) + t_hp) / t_hp
            points.append({"d": d, "hp_turnaround_fifo_us": round(res["fifo"], 3) if res["fifo"] else None,
                           "hp_turnaround_flep_us": round(res["flep"], 3) if res["flep"] else None,
                           "speedup": round(res["fifo"] / res["flep"], 3) if res["fifo"] and res["flep"] else None,
                           "zero_overhead_bound": round(bound, 3)})
    parity = spot_parity(wl, torch)
    rt.close()
    sp = [p["speedup"] for p in points if p["speedup"]]
    out = {"metric": METRIC, "value": round(float(np.mean(sp)), 3) if sp else None, "unit": "x",
           "value_definition": "HP turnaround speedup FIFO / FLEP averaged over arrival points d = 0.1..0.9 of the LP",
           "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "higher_is_better": True,
           "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic (seeded; synth/gen.py)",
           "config": {"workload": "LP SpMV-CSR 2^20 rows (counter worker, C=K=1), HP stencil5 4096^2 (CLC), "
                                  "HP arrival = device trigger at block d*N of the LP", "reps_per_point": reps,
                      "l2": "flushed before every step"},
           "standalone_us": {"lp": round(t_lp, 3), "hp": round(t_hp, 3)},
           "points": points, "parity": parity, "clocks": clk.summary()}
    _emit(out, rank, args)
    barrier(world)
    return out


# ------------------------------------------------------------------------------------------
def assign_jobs(jobs, t_e_of, world):
    """One job queue feeding `world` independent per-GPU schedulers (configs[4]): each arrival
    goes to the GPU whose predicted backlog (sum of T_e of the work assigned to it that is not
    yet predicted to be done) ends first; ties -> lowest index. Deterministic, so every rank
    computes the same partition without communication. Returns one job list per GPU."""
    backlog_end = [0] * world
    out = [[] for _ in range(world)]
    for j in jobs:
        avail = [max(b, j["arrival_ns"]) for b in backlog_end]
        r = min(range(world), key=lambda i: (avail[i], i))
        backlog_end[r] = avail[r] + int(t_e_of(j))
        out[r].append(j)
    return out


def _agree_t_alone(t_alone, world, torch):
    """Every rank must partition the job queue identically (assign_jobs is deterministic in its
    inputs): use the mean over ranks of the measured standalone times."""
    if world == 1:
        return t_alone
    from bench import allreduce_mean
    keys = sorted(t_alone)
    vals = allreduce_mean([float(t_alone[k]) for k in keys], world, torch)
    return {k: int(round(v)) for k, v in zip(keys, vals)}


QUEUE_CHUNK = {"saxpy_f32": (8, False), "spmv": (2, True), "stencil_f32": (2, True), "gemm_bf16": (1, False)}
# FLEP_QUEUE_FETCH=spec (the default): SpMV and stencil fetch their C-block chunks speculatively
# (R34) instead of prefetching them: a prefetching worker runs the chunk it holds before it yields
# (A4), which doubles its drain; a speculative fetch hands that chunk back through the worker's
# record. Measured on configs[4] (profiles/r02_queue_fetch_spec.jsonl): preemption latency p99
# 45-46 -> 27.7 us (SpMV 2^23 victims p50 38 -> 22-24 us), same throughput and overheads.
# FLEP_QUEUE_FETCH=prefetch restores the round-1/2 setting (QUEUE_CHUNK).
QUEUE_CHUNK_SPEC = {"saxpy_f32": (8, False), "spmv": (2, False), "stencil_f32": (2, False), "gemm_bf16": (1, False)}


def _qopts(F, ty, body):
    """register_kernel options of a queue kernel of type `ty` (configs[3], configs[4], E13)."""
    spec = os.environ.get("FLEP_QUEUE_FETCH", "spec") == "spec"
    C, pf = (QUEUE_CHUNK_SPEC if spec else QUEUE_CHUNK)[ty]
    gemm = body in (F.BODY_GEMM_BF16, F.BODY_GEMM_BF16_2SM, F.BODY_GEMM_BF16_2SM_W)
    if ty == "stencil_f32" and os.environ.get("FLEP_QUEUE_STENCIL") == "clc":
        # experiment: the stencil victims on the CLC fetch at C = K = 1 (the barrier-free form, R38)
        return dict(chunk=1, poll=1, clc=True)
    return dict(chunk=C, poll=1, prefetch=pf, spec_fetch=spec and not gemm and ty != "saxpy_f32", in_tile=gemm)


def _queue_instances(torch, F, seed):
    """Device inputs for every (type, size class) of config 4 (seeded torch generators)."""
    from synth.gen import QUEUE_SIZES
    g = torch.Generator(device="cuda")
    g.manual_seed(seed)
    inst = {}
    for ty, sizes in QUEUE_SIZES.items():
        for cls, sz in enumerate(sizes):
            if ty == "saxpy_f32":
                x = torch.rand(sz, device="cuda", generator=g)
                y = torch.rand(sz, device="cuda", generator=g)
                inst[(ty, cls)] = (F.BODY_SAXPY_F32, F.saxpy_grid(sz), F.saxpy_f32_args(y, x, 0.5), (x, y),
                                   12 * sz)
            elif ty == "spmv":
                lens = torch.randint(0, 21, (sz,), device="cuda", generator=g)
                rowptr = torch.zeros(sz + 1, dtype=torch.int64, device="cuda")
                rowptr[1:] = torch.cumsum(lens, 0)
                nnz = int(rowptr[-1])
                cols = torch.randint(0, sz, (nnz,), device="cuda", generator=g)
                rows = torch.repeat_interleave(torch.arange(sz, device="cuda"), lens)
                key, _ = torch.sort(rows * sz + cols)
                col = (key % sz).to(torch.int32)
                val = torch.rand(nnz, device="cuda", generator=g) * 2 - 1
                xv = torch.rand(sz, device="cuda", generator=g) * 2 - 1
                yv = torch.empty(sz, device="cuda")
                rp = rowptr.to(torch.int32)
                inst[(ty, cls)] = (F.BODY_SPMV_CSR_F32, F.spmv_grid(sz), F.spmv_args(yv, rp, col, val, xv),
                                   (rp, col, val, xv, yv), 8 * nnz + 12 * sz)
            elif ty == "stencil_f32":
                a = torch.rand(sz, sz, device="cuda", generator=g)
                o = torch.empty_like(a)
                inst[(ty, cls)] = (F.BODY_STENCIL5_F32, F.stencil_grid(sz), F.stencil_args(o, a), (a, o), 8 * sz * sz)
            else:
                A = (torch.rand(sz, sz, device="cuda", generator=g) * 2 - 1).to(torch.bfloat16)
                B = (torch.rand(sz, sz, device="cuda", generator=g) * 2 - 1).to(torch.bfloat16)
                C = torch.empty(sz, sz, device="cuda", dtype=torch.bfloat16)
                # FLEP_QUEUE_GEMM: 1 the 1-CTA body, 2 the CTA-pair body (R32), 3 its wide tile
                which = os.environ.get("FLEP_QUEUE_GEMM", "1")
                inst[(ty, cls)] = {"1": (F.BODY_GEMM_BF16, F.gemm_grid(sz, sz)),
                                   "2": (F.BODY_GEMM_BF16_2SM, F.gemm2_grid(sz, sz)),
                                   "3": (F.BODY_GEMM_BF16_2SM_W, F.gemm2w_grid(sz, sz))}[which] + (
                                       F.gemm_args(C, A, B), (A, B, C), 2 * sz ** 3)
    return inst


def _run_trace(F, torch, local, policy, trace, inst, t_alone, overhead_ns, streams, slice_blocks=0,
               want_lat=False):
    rt = F.Runtime(device=local, policy=policy, slice_blocks=slice_blocks)
    kid = {}
    used = {(j["type"], j["size_class"]) for j in trace}
    for key, (body, grid, a, keep, _) in inst.items():
        if key not in used:
            continue
        kid[key] = rt.register_kernel(body, name=f"{key[0]}-{key[1]}", model=(0, 0, 0, 0, float(t_alone[key])),
                                      overhead_ns=int(overhead_ns), **_qopts(F, key[0], body))
    hs = []
    call_ns = []
    _run_trace.lat_keys = []           # victim kernel of each latency sample (want_lat)
    t0 = F.now_ns() + 2_000_000
    for i, job in enumerate(trace):
        key = (job["type"], job["size_class"])
        body, grid, a, keep, _ = inst[key]
        target = t0 + job["arrival_ns"]
        while F.now_ns() < target:
            pass
        tl = F.now_ns()
        hs.append((rt.launch(kid[key], grid, a, priority=job["priority"], stream=streams[i % len(streams)]), key))
        call_ns.append(F.now_ns() - tl)
    for h, _ in hs:
        rt.sync(h, timeout_ns=60_000_000_000)
    turn = []
    lat = []
    for h, key in hs:
        info = rt.query(h)
        turn.append((info.t_finish - info.t_arrive, key, info.t_arrive - t0, info.t_first_start - t0,
                     info.t_finish - t0, info.epoch))
        # host-observed preemption latency of the last drained epoch (request -> drained status)
        if info.epoch >= 2 and info.t_last_drain > 0 and info.t_last_request > 0:
            lat.append((info.t_last_drain - info.t_last_request) / 1e3)
            _run_trace.lat_keys.append(f"{key[0]}-{key[1]}")
    dec = rt.decision_log()
    evl = rt.event_log()
    rt.close()
    _run_trace.last_call_us = {"mean": round(float(np.mean(call_ns)) / 1e3, 2), "max": round(float(np.max(call_ns)) / 1e3, 2)}
    if want_lat:
        return turn, dec, evl, lat
    return turn, dec, evl


def _measure_t_alone(F, torch, local, inst):
    """Standalone turnaround (ns) of every queue instance through the same runtime path (FIFO, idle
    GPU, L2 flushed: the queue interleaves working sets); median of 3 after one warm-up."""
    from bench import L2Flush
    flush = L2Flush(torch)
    t_alone = {}
    rt = F.Runtime(device=local, policy=F.POLICY_FIFO)
    for key, (body, grid, a, keep, _) in inst.items():
        k = rt.register_kernel(body, **_qopts(F, key[0], body))
        ts = []
        for r in range(4):
            flush.zero_()
            torch.cuda.synchronize()
            h = rt.launch(k, grid, a)
            rt.sync(h)
            info = rt.query(h)
            if r:
                ts.append(info.t_finish - info.t_arrive)
        t_alone[key] = int(np.median(ts))
    rt.close()
    del flush
    return t_alone


def run_queue(args, rank, world, local):
    """configs[3] (and configs[4] at N > 1): same-priority mixed queue of 64 kernels (SAXPY-f32,
    SpMV, stencil5, bf16 GEMM up to 8192^3) with Poisson arrivals at offered load rho; ANTT and
    STP for FIFO (MPS-like co-run baseline), FLEP-HPF (SRPT + overhead, Fig. 6) and kernel
    slicing; NATT gain = ANTT_base / ANTT_FLEP. At N > 1 one job queue of
    64*N kernels feeds N independent per-GPU schedulers (least predicted backlog)."""
    import torch
    import bench_check as M
    from bench import barrier
    from paper_conf_asplos_wulzj17_b200 import flep as F
    torch.cuda.set_device(local)
    inst = _queue_instances(torch, F, seed=5)
    streams = [torch.cuda.Stream() for _ in range(4)]
    t_alone = _agree_t_alone(_measure_t_alone(F, torch, local, inst), world, torch)
    n_total = args.queue_kernels * world
    mean_alone = float(np.mean([t_alone[(j["type"], j["size_class"])]
                                for j in gen.queue_trace(5, n_total, 1)]))
    gap = int(mean_alone / args.rho)
    full = gen.queue_trace(6 if world > 1 else 5, n_total, gap)
    mine = assign_jobs(full, lambda j: t_alone[(j["type"], j["size_class"])], world)[rank]
    overhead_ns = 20_000
    res = {}
    debug = {}
    logs = {}
    # untimed warm-up of a short prefix (first-use costs of a fresh runtime, stream and event pools)
    _run_trace(F, torch, local, F.POLICY_FIFO, mine[:8], inst, t_alone, overhead_ns, streams)
    for name, pol in (("FIFO", F.POLICY_FIFO), ("HPF", F.POLICY_HPF), ("SLICE", F.POLICY_SLICE),
                      ("SLICE_DEVICE", F.POLICY_SLICE_DEVICE), ("REORDER", F.POLICY_REORDER)):
        turn, dec, evl = _run_trace(F, torch, local, pol, mine, inst, t_alone, overhead_ns, streams)
        tt = [t[0] for t in turn]
        al = [t_alone[t[1]] for t in turn]
        debug[name] = [(f"{t[1][0]}-{t[1][1]}", t[2], t[3], t[4], t[5], t_alone[t[1]]) for t in turn]
        res[name] = {"antt": M.antt(tt, al), "stp": M.stp(tt, al), "preemptions": sum(1 for d in dec if d[1] == 2),
                     "makespan_ms": round(max(t[4] for t in turn) / 1e6, 3)}
        logs[name] = {"events": [list(map(int, e)) for e in evl], "decisions": [list(map(int, d_)) for d_ in dec]}
        res[name]["launch_call_us"] = _run_trace.last_call_us
    # the runtime's event and decision logs (replayed through the oracle DES by
    # tests/test_policy_replay.py from the committed copy under tests/golden/)
    import os
    ev_dir = os.environ.get("FLEP_EVIDENCE_DIR")
    if ev_dir and rank == 0:
        with open(os.path.join(ev_dir, "queue_logs.json"), "w") as fh:
            json.dump({"workload": "configs[3] queue, seed 5", "logs": logs}, fh)
    gain_fifo = res["FIFO"]["antt"] / res["HPF"]["antt"]
    gain_slice = res["SLICE"]["antt"] / res["HPF"]["antt"]
    gain_slice_dev = res["SLICE_DEVICE"]["antt"] / res["HPF"]["antt"]
    out = {"metric": METRIC, "value": round(gain_fifo, 3), "unit": "x (ANTT_FIFO / ANTT_FLEP)",
           "value_definition": "co-run NATT gain of FLEP-HPF over the FIFO (MPS-like) baseline on the same trace",
           "n_gpus": world, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
           "dtype": "mixed (f32, bf16->f32)", "data": "synthetic (seeded)",
           "config": {"workload": f"configs[{3 if world == 1 else 4}]: same-priority queue of {n_total} kernels "
                                  f"(SAXPY-f32/SpMV/stencil5/GEMM-bf16 x trivial/small/large, up to 8192^3), "
                                  f"Poisson arrivals rho={args.rho}", "kernels_this_gpu": len(mine),
                      "mean_gap_us": round(gap / 1e3, 1), "overhead_estimate_ns": overhead_ns},
           "antt": {k: round(v["antt"], 3) for k, v in res.items()},
           "stp": {k: round(v["stp"], 3) for k, v in res.items()},
           "preemptions": {k: v["preemptions"] for k, v in res.items()},
           "natt_gain_vs_fifo": round(gain_fifo, 3), "natt_gain_vs_slicing": round(gain_slice, 3),
           "natt_gain_vs_slicing_device": round(gain_slice_dev, 3),
           "slicing_note": "SLICE = host-issued slices, at most two in flight (R19); SLICE_DEVICE = every slice "
                           "enqueued at launch with the device check at slice entry (R31)",
           "reordering_gain_vs_fifo": round(res["FIFO"]["antt"] / res["REORDER"]["antt"], 3),
           "stp_degradation_vs_fifo": round(1 - res["HPF"]["stp"] / res["FIFO"]["stp"], 4),
           "replay_parity": "checked on CPU: tests/test_policy_replay.py replays the committed logs (tests/golden/queue_logs_r01.json) through the oracle DES",
           "makespan_ms": {k: v["makespan_ms"] for k, v in res.items()},
           "launch_call_us": {k: v["launch_call_us"] for k, v in res.items()},
           "launch_call_note": "host time of the flep_launch call; SLICE_DEVICE enqueues every slice in that call "
                               "(up to ~110 kernel launches, ~4 us each), which is its max; FLEP_DEBUG_SLOW=<us> "
                               "prints any slower epoch start with its materialize/launch split",
           "t_alone_us": {f"{k[0]}-{k[1]}": round(v / 1e3, 1) for k, v in sorted(t_alone.items())}}
    if world > 1:
        from bench import allreduce_max
        out["value"] = round(-allreduce_max([-gain_fifo], world, torch)[0], 3)
        out["value_definition"] += " (min over GPUs)"
    _emit(out, rank, args)
    if rank == 0:
        import os
        dbg = os.environ.get("FLEP_EVIDENCE_DIR")
        if dbg:
            with open(os.path.join(dbg, "queue_debug.json"), "w") as fh:
                json.dump(debug, fh)
    barrier(world)
    return out


# ------------------------------------------------------------------------------------------
CORUN_TYPES = ("saxpy_f32", "spmv", "stencil_f32", "gemm_bf16")
CORUN_SHORT = {"saxpy_f32": "VA", "spmv": "SPMV", "stencil_f32": "ST", "gemm_bf16": "MM"}


def corun_cases(seed=7, n_triplets=28, gap_ns=20_000):
    """The paper's co-run experiments as job traces over the queue instances (large = class 2,
    small = class 1): E4 (Fig. 8) every large low-priority kernel with every small
    high-priority kernel launched right after it; E6/E7 (Figs. 10-11) the same pairs at
    equal priority; E8 (Fig. 12) 28 seeded triplets A_B_C, A large then B and C small
    (B != C). Returns [(experiment, name, trace)]."""
    cases = []
    for lp in CORUN_TYPES:
        for hp in CORUN_TYPES:
            for exp, prio in (("E4", 1), ("E6", 0)):
                cases.append((exp, f"{CORUN_SHORT[lp]}_{CORUN_SHORT[hp]}", [
                    {"id": 0, "type": lp, "size_class": 2, "priority": 0, "arrival_ns": 0},
                    {"id": 1, "type": hp, "size_class": 1, "priority": prio, "arrival_ns": gap_ns}]))
    # the paper's named triplet VA_SPMV_MM and n_triplets - 1 seeded others
    named = ("saxpy_f32", "spmv", "gemm_bf16")
    trip = [(a, b, c) for a in CORUN_TYPES for b in CORUN_TYPES for c in CORUN_TYPES if b != c and (a, b, c) != named]
    g = gen.rng(seed)
    pick = [trip[i] for i in g.choice(len(trip), size=n_triplets - 1, replace=False).tolist()] + [named]
    for a, b, c in sorted(pick, key=lambda t: tuple(CORUN_TYPES.index(x) for x in t)):
        cases.append(("E8", f"{CORUN_SHORT[a]}_{CORUN_SHORT[b]}_{CORUN_SHORT[c]}", [
            {"id": 0, "type": a, "size_class": 2, "priority": 0, "arrival_ns": 0},
            {"id": 1, "type": b, "size_class": 1, "priority": 0, "arrival_ns": gap_ns},
            {"id": 2, "type": c, "size_class": 1, "priority": 0, "arrival_ns": 2 * gap_ns}]))
    return cases


def run_coruns(args, rank, world, local):
    """The paper's co-run matrices on one B200 through the managed runtime: E4 high-priority
    speedup (Fig. 8: HP turnaround under the FIFO / MPS-like default co-run over FLEP-HPF), E6
    ANTT gain and E7 STP degradation of equal-priority pairs (Figs. 10-11), E8 ANTT gain of 28
    triplets and of non-preemptive reordering (Fig. 12). Median of `reps` runs per case and
    policy; the runtime's event and decision logs of the first run of every case are written to
    FLEP_EVIDENCE_DIR (corun_logs.json) for the oracle replay test."""
    import os
    import torch
    import bench_check as M
    from bench import ClockSampler, barrier, physical_gpu_index
    from paper_conf_asplos_wulzj17_b200 import flep as F
    torch.cuda.set_device(local)
    inst = _queue_instances(torch, F, seed=5)
    inst = {k: v for k, v in inst.items() if k[1] >= 1}          # small and large classes only
    streams = [torch.cuda.Stream() for _ in range(4)]
    t_alone = _measure_t_alone(F, torch, local, inst)
    overhead_ns = 20_000
    reps = max(1, int(getattr(args, "corun_reps", 3)))
    cases = corun_cases()
    pols = {"E4": (("FIFO", F.POLICY_FIFO), ("HPF", F.POLICY_HPF)),
            "E6": (("FIFO", F.POLICY_FIFO), ("HPF", F.POLICY_HPF)),
            "E8": (("FIFO", F.POLICY_FIFO), ("HPF", F.POLICY_HPF), ("REORDER", F.POLICY_REORDER))}
    _run_trace(F, torch, local, F.POLICY_HPF, cases[0][2], inst, t_alone, overhead_ns, streams)   # warm-up
    rows, logs = [], {}
    with ClockSampler(physical_gpu_index(local)) as clk:
        for exp, name, trace in cases:
            row = {"exp": exp, "case": name}
            for pname, pol in pols[exp]:
                turns = []
                for r in range(reps):
                    turn, dec, evl = _run_trace(F, torch, local, pol, trace, inst, t_alone, overhead_ns, streams)
                    turns.append([t[0] for t in turn])
                    if r == 0:
                        logs[f"{exp}/{name}/{pname}"] = {"events": [list(map(int, e)) for e in evl],
                                                         "decisions": [list(map(int, d_)) for d_ in dec]}
                tt = [int(np.median([t[i] for t in turns])) for i in range(len(trace))]
                al = [t_alone[(j["type"], j["size_class"])] for j in trace]
                row[pname] = {"turn_us": [round(x / 1e3, 1) for x in tt], "antt": round(M.antt(tt, al), 3),
                              "stp": round(M.stp(tt, al), 3)}
            al = [t_alone[(j["type"], j["size_class"])] for j in trace]
            if exp == "E4":
                row["hp_speedup"] = round(row["FIFO"]["turn_us"][1] / row["HPF"]["turn_us"][1], 2)
                # a non-preemptive co-run makes the HP wait for the rest of the LP (P:321's bound)
                row["hp_speedup_bound"] = round((al[0] - trace[1]["arrival_ns"] + al[1]) / al[1], 2)
            else:
                row["antt_gain"] = round(row["FIFO"]["antt"] / row["HPF"]["antt"], 2)
                row["stp_degradation"] = round(1 - row["HPF"]["stp"] / row["FIFO"]["stp"], 4)
                if exp == "E8":
                    row["reorder_gain"] = round(row["FIFO"]["antt"] / row["REORDER"]["antt"], 3)
            rows.append(row)
    ev_dir = os.environ.get("FLEP_EVIDENCE_DIR")
    if ev_dir and rank == 0:
        with open(os.path.join(ev_dir, "corun_logs.json"), "w") as fh:
            json.dump({"workload": "co-run matrices E4/E6/E8 over the queue instances (seed 5)", "logs": logs}, fh)

    def summ(exp, key):
        v = [r[key] for r in rows if r["exp"] == exp]
        return {"mean": round(float(np.mean(v)), 3), "min": round(float(np.min(v)), 3),
                "max": round(float(np.max(v)), 3), "n": len(v),
                "argmax": max((r for r in rows if r["exp"] == exp), key=lambda r: r[key])["case"]}
    out = {"metric": METRIC, "value": summ("E6", "antt_gain")["mean"], "unit": "x (ANTT_FIFO / ANTT_FLEP)",
           "value_definition": "mean ANTT gain of FLEP-HPF over the FIFO (MPS-like) co-run over the 16 "
                               "equal-priority pairs (E6, Fig. 10)",
           "n_gpus": world, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
           "dtype": "mixed (f32, bf16->f32)", "data": "synthetic (seeded)",
           "config": {"workload": "co-runs of the configs[3] instances: large = class 2 (SAXPY 2^28, SpMV 2^23 rows, "
                                  "stencil 16384^2, GEMM 8192^3), small = class 1 (2^24, 2^20 rows, 4096^2, 4096^3); "
                                  "the second (and third) kernel arrives 20 (40) us after the first",
                      "reps": reps, "overhead_estimate_ns": overhead_ns},
           "E4_hp_speedup": summ("E4", "hp_speedup"), "E6_antt_gain": summ("E6", "antt_gain"),
           "E7_stp_degradation": summ("E6", "stp_degradation"), "E8_antt_gain": summ("E8", "antt_gain"),
           "E8_reorder_gain": summ("E8", "reorder_gain"),
           "paper": "K40: E4 10.1x mean / 24.2x max / 4.1x min; E6 8x mean, 27x max; E7 5.4 %; E8 6.6x mean, "
                    "20.2x max (VA_SPMV_MM); reordering 2.3 % (P:321, P:329, P:343, P:349-351)",
           "t_alone_us": {f"{k[0]}-{k[1]}": round(v / 1e3, 1) for k, v in sorted(t_alone.items())},
           "cases": rows, "clocks": clk.summary()}
    _emit(out, rank, args)
    barrier(world)
    return out


def run_ffs(args, rank, world, local):
    """FFS experiment (Figs. 13-14): two applications keep invoking the
    same long kernel (SAXPY-int32 over 2^30 elements, ~2 ms) in a loop, priorities 1 and 0 (weights
    2:1), max_overhead = 10%. Reports each application's GPU share and the throughput
    degradation against one application running alone."""
    import threading

    import torch
    from bench import barrier
    from paper_conf_asplos_wulzj17_b200 import flep as F
    torch.cuda.set_device(local)
    n = 1 << 30
    dur = args.ffs_seconds
    bufs = [(torch.ones(n, dtype=torch.int32, device="cuda"), torch.ones(n, dtype=torch.int32, device="cuda"))
            for _ in range(2)]

    def loop(rt, k, app, prio, stop_at, counts):
        x, y = bufs[app]
        s = torch.cuda.Stream()
        while F.now_ns() < stop_at:
            h = rt.launch(k, F.saxpy_grid(n), F.saxpy_i32_args(y, x, 1), priority=prio, stream=s)
            rt.sync(h, timeout_ns=5_000_000_000)
            if F.now_ns() <= stop_at:
                counts[app] += 1

    def run(policy, apps):
        rt = F.Runtime(device=local, policy=policy, max_overhead_ppm=100_000)
        k = rt.register_kernel(F.BODY_SAXPY_I32, chunk=8, poll=1, overhead_ns=10_000,
                               model=(0, 0, 0, 0, 2_000_000))
        counts = [0, 0]
        stop_at = F.now_ns() + int(dur * 1e9)
        th = [threading.Thread(target=loop, args=(rt, k, a, 1 - a, stop_at, counts)) for a in apps]
        for t_ in th:
            t_.start()
        for t_ in th:
            t_.join()
        dec = rt.decision_log()
        evl = rt.event_log()
        rt.close()
        import os
        dbg = os.environ.get("FLEP_EVIDENCE_DIR")
        if dbg and policy == F.POLICY_FFS:
            with open(os.path.join(dbg, "ffs_debug.json"), "w") as fh:
                json.dump({"decisions": dec[-600:], "events": evl[-600:], "n_dec": len(dec), "n_ev": len(evl)}, fh)
        return counts, sum(1 for d in dec if d[1] == 2)

    alone, _ = run(F.POLICY_FIFO, [0])
    shared, npre = run(F.POLICY_FFS, [0, 1])
    tot = shared[0] + shared[1]
    out = {"metric": METRIC, "value": round(shared[0] / tot, 4) if tot else None, "unit": "GPU share of the weight-2 app",
           "value_definition": "FFS GPU share of the high-priority (weight 2) application; target 2/3 (P:363)",
           "n_gpus": world, "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32",
           "data": "synthetic", "config": {"workload": "FFS pair: SAXPY-int32 2^30 invoked in a loop by two applications "
                                                      "(priorities 1, 0), max_overhead 10%", "seconds": dur},
           "kernels_completed": {"weight2": shared[0], "weight1": shared[1], "alone": alone[0]},
           "share_weight1": round(shared[1] / tot, 4) if tot else None,
           "throughput_degradation": round(1 - tot / alone[0], 4) if alone[0] else None,
           "preemptions": npre}
    _emit(out, rank, args)
    barrier(world)
    return out


# ------------------------------------------------------------------------------------------
def run_model(args, rank, world, local):
    """Offline phase (§4.2; Fig. 7): fit each body's duration model on
    random inputs (100 per body), report the prediction error on held-out inputs, and the
    profiled preemption overhead O."""
    import torch
    from bench import L2Flush, barrier
    from paper_conf_asplos_wulzj17_b200 import calibrate, flep as F
    torch.cuda.set_device(local)
    wl = calibrate.Workloads(torch, seed=11 + rank)
    fl = L2Flush(torch)
    rt = F.Runtime(device=local, policy=F.POLICY_FIFO)
    rows = {}
    bodies = {"saxpy_f32": (F.BODY_SAXPY_F32, 8, False), "spmv": (F.BODY_SPMV_CSR_F32, 2, True),
              "stencil_f32": (F.BODY_STENCIL5_F32, 2, True), "gemm_bf16": (F.BODY_GEMM_BF16, 1, False)}
    for name, (body, chunk, pf) in bodies.items():
        model, X, y = calibrate.fit_duration_model(rt, torch, wl, body, n_train=args.model_train, chunk=chunk,
                                                   prefetch=pf, flush=fl.zero_)
        k = rt.register_kernel(body, chunk=chunk, poll=1, prefetch=pf)
        errs = []
        for _ in range(args.model_test):
            grid, a, feats = wl.case(body, wl.random_size(body))
            t = calibrate.measure_duration(rt, k, grid, a, torch, fl.zero_, reps=1)
            errs.append(abs(float(calibrate.predict(model, feats)) - t) / t)
        size = {F.BODY_SAXPY_F32: 1 << 26, F.BODY_SPMV_CSR_F32: 1 << 22, F.BODY_STENCIL5_F32: 8192,
                F.BODY_GEMM_BF16: 4096}[body]
        o, t_alone = calibrate.preemption_overhead(torch, wl, body, size, runs=args.overhead_runs, chunk=chunk,
                                                   prefetch=pf, flush=fl.zero_)
        rows[name] = {"model": [round(v, 6) for v in model], "mean_abs_pct_error": round(100 * float(np.mean(errs)), 2),
                      "max_abs_pct_error": round(100 * float(np.max(errs)), 2), "train": len(y), "test": len(errs),
                      "preempt_overhead_ns": o, "overhead_reference_size": size,
                      "standalone_span_us": round(t_alone / 1e3, 2)}
    rt.close()
    mean_err = float(np.mean([r["mean_abs_pct_error"] for r in rows.values()]))
    out = {"metric": METRIC, "value": round(mean_err, 2), "unit": "% mean abs duration-prediction error",
           "value_definition": "ridge duration model (P:192) on held-out random inputs, mean over bodies (paper: 6.9 % on K40)",
           "n_gpus": world, "higher_is_better": False, "scaling": "weak", "vs_baseline": None, "dtype": "mixed",
           "data": "synthetic (seeded)", "config": {"workload": "offline phase: model fit + O profiling per body",
                                                      "train_per_body": args.model_train, "test_per_body": args.model_test},
           "bodies": rows}
    _emit(out, rank, args)
    barrier(world)
    return out


# ------------------------------------------------------------------------------------------
def run_tune(args, rank, world, local):
    """Offline tuning of the amortizing factor L = C*K (the smallest L, tried from small
    to large, whose overhead is under 4 %) for every body at the BASELINE configs' sizes."""
    import torch
    from bench import L2Flush, barrier
    from paper_conf_asplos_wulzj17_b200 import calibrate, flep as F
    torch.cuda.set_device(local)
    rt = F.Runtime(device=local, exec_on_user_stream=True)
    fl = L2Flush(torch)
    T = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()  # noqa: E731
    g = torch.Generator(device="cuda")
    g.manual_seed(21 + rank)
    cases = {}
    x, y = gen.saxpy_i32_inputs(1 << 20, seed=1)
    keep = [T(y), T(x)]                  # device tensors must outlive the args structs (raw pointers)
    cases["saxpy_i32_2^20 (configs[0] LP)"] = (F.BODY_SAXPY_I32, F.saxpy_grid(1 << 20), F.saxpy_i32_args(keep[0], keep[1], 3))
    xs = torch.ones(1 << 28, dtype=torch.int32, device="cuda")
    ys = torch.ones(1 << 28, dtype=torch.int32, device="cuda")
    cases["saxpy_i32_2^28"] = (F.BODY_SAXPY_I32, F.saxpy_grid(1 << 28), F.saxpy_i32_args(ys, xs, 3))
    rp, col, val, xv = gen.csr_inputs(1 << 20, seed=2)
    yv = torch.zeros(1 << 20, device="cuda")
    keep += [T(rp), T(col), T(val), T(xv)]
    cases["spmv_2^20 (configs[1] LP)"] = (F.BODY_SPMV_CSR_F32, F.spmv_grid(1 << 20),
                                          F.spmv_args(yv, *keep[2:6]))
    st = T(gen.stencil_f32_input(4096, seed=3))
    so = torch.empty_like(st)
    cases["stencil_4096^2 (configs[1] HP)"] = (F.BODY_STENCIL5_F32, F.stencil_grid(4096), F.stencil_args(so, st))
    sb = torch.rand(16384, 16384, device="cuda", generator=g)
    sbo = torch.empty_like(sb)
    cases["stencil_16384^2 (configs[2])"] = (F.BODY_STENCIL5_F32, F.stencil_grid(16384), F.stencil_args(sbo, sb))
    A = (torch.rand(8192, 8192, device="cuda", generator=g) * 2 - 1).to(torch.bfloat16)
    B = (torch.rand(8192, 8192, device="cuda", generator=g) * 2 - 1).to(torch.bfloat16)
    Cm = torch.empty(8192, 8192, device="cuda", dtype=torch.bfloat16)
    cases["gemm_8192^3 (configs[3])"] = (F.BODY_GEMM_BF16, F.gemm_grid(8192, 8192), F.gemm_args(Cm, A, B))
    rows = {}
    for name, (body, grid, a) in cases.items():
        choice, table = calibrate.tune_amortizing_factor(rt, torch, body, grid, a, fl.zero_, bound=args.tune_bound,
                                                         reps=args.reps)
        rows[name] = {"choice": {k: (round(v, 4) if isinstance(v, float) else v) for k, v in choice.items()},
                      "tried": len(table),
                      "table": [{k: (round(v, 4) if isinstance(v, float) else v) for k, v in r.items()} for r in table]}
    rt.close()
    met = sum(1 for r in rows.values() if r["choice"]["met"])
    out = {"metric": METRIC, "value": met, "unit": f"kernels (of {len(rows)}) whose tuned L meets the overhead bound",
           "value_definition": "offline amortizing-factor tuning (P:166): smallest L = C*K with wrapped/unwrapped - 1 "
                               f"< {args.tune_bound} (event-timed, L2 flushed, trimmed mean of {args.reps})",
           "n_gpus": world, "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "mixed",
           "data": "synthetic (seeded)", "config": {"workload": "amortizing-factor tuning at the BASELINE configs' sizes",
                                                      "bound": args.tune_bound},
           "kernels": rows}
    _emit(out, rank, args)
    barrier(world)
    return out


# ------------------------------------------------------------------------------------------
SCALE_PRED_US = {"saxpy_f32": (4.0, 30.0, 420.0), "spmv": (8.0, 62.0, 520.0),
                 "stencil_f32": (5.0, 24.0, 330.0), "gemm_bf16": (16.0, 95.0, 700.0)}


def run_scale_dry(args, rank, world, local):
    """configs[4] control flow without CUDA (bench.py --dry-run, CPU gloo): the launcher, the
    process group, the deterministic job partition of one 512-kernel queue over `world` per-GPU
    schedulers, the gather and rank 0's single JSON line. Standalone times are the fixed
    predictions above instead of measurements."""
    from bench import barrier, gather_objects
    t_e = {(ty, c): int(v[c] * 1e3) for ty, v in SCALE_PRED_US.items() for c in range(3)}
    n_total = args.scale_kernels
    mean_alone = float(np.mean([t_e[(j["type"], j["size_class"])] for j in gen.queue_trace(6, n_total, 1)]))
    gap = int(mean_alone / (args.rho * world))
    full = gen.queue_trace(6, n_total, gap)
    parts = assign_jobs(full, lambda j: t_e[(j["type"], j["size_class"])], world)
    mine = parts[rank]
    rec = {"rank": rank, "local_rank": local, "kernels": len(mine), "ids": [j["id"] for j in mine],
           "predicted_busy_us": round(sum(t_e[(j["type"], j["size_class"])] for j in mine) / 1e3, 1)}
    allr = gather_objects(rec, world)
    ids = sorted(i for r in allr for i in r["ids"])
    out = {"metric": METRIC, "value": None, "unit": "us", "n_gpus": world, "dry_run": True,
           "higher_is_better": False, "scaling": "weak", "vs_baseline": None, "dtype": "n/a", "data": "synthetic",
           "config": {"workload": f"configs[4]: one job queue of {n_total} mixed kernels over {world} per-GPU "
                                  "schedulers (dry run: no CUDA)", "parallelism": f"replicas x{world}",
                      "mean_gap_us": round(gap / 1e3, 2)},
           "ranks": [{k: v for k, v in r.items() if k != "ids"} for r in allr],
           "partition_ok": ids == list(range(n_total)),
           "backend": _backend(world)}
    _emit(out, rank, args)
    barrier(world)
    return out


def _backend(world):
    if world == 1:
        return None
    import torch.distributed as dist
    return dist.get_backend()


def run_scale_queue(args, rank, world, local):
    """configs[4]: N x B200 independent per-GPU schedulers (one FLEP runtime each, HPF) fed from
    one job queue of 512 mixed kernels (SAXPY-f32 / SpMV / stencil5 / bf16 GEMM, trivial / small /
    large, seed 6), Poisson arrivals at offered load rho per GPU; each arrival goes to the GPU with
    the least predicted backlog (assign_jobs, deterministic on every rank). Reports the wrapper
    overhead of every instance (wrapped vs unwrapped, CUDA events), the per-GPU preemption-latency
    distribution (host-observed request -> drained epoch of every SRPT preemption), ANTT of
    FLEP-HPF vs FIFO over all kernels, and aggregate throughput (kernels / s over the slowest GPU's
    makespan). There is no collective on the data path: the process group only
    carries the standalone-time agreement and the final gather."""
    import torch
    import bench_check as M
    from bench import ClockSampler, L2Flush, barrier, gather_objects, physical_gpu_index
    from paper_conf_asplos_wulzj17_b200 import flep as F
    torch.cuda.set_device(local)
    inst = _queue_instances(torch, F, seed=5)
    streams = [torch.cuda.Stream() for _ in range(4)]
    flush = L2Flush(torch)
    S = torch.cuda.Stream()
    t_alone, over = {}, {}
    rt = F.Runtime(device=local, policy=F.POLICY_FIFO)
    rt_m = F.Runtime(device=local, exec_on_user_stream=True)
    for key, (body, grid, a, keep, _) in sorted(inst.items()):
        k = rt.register_kernel(body, **_qopts(F, key[0], body))
        ts = []
        for r in range(3):
            flush.zero_()
            torch.cuda.synchronize()
            h = rt.launch(k, grid, a)
            rt.sync(h)
            info = rt.query(h)
            if r:
                ts.append(info.t_finish - info.t_arrive)
        t_alone[key] = int(np.median(ts))
        km = rt_m.register_kernel(body, **_qopts(F, key[0], body))
        tw, tu = [], []
        for r in range(4):
            for mode in ("w", "u"):
                with torch.cuda.stream(S):
                    flush.zero_()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(S)
                if mode == "w":
                    h = rt_m.launch(km, grid, a, stream=S)
                else:
                    rt_m.launch_unwrapped(body, grid, a, stream=S)
                e1.record(S)
                e1.synchronize()
                if mode == "w":
                    rt_m.sync(h)
                if r:
                    (tw if mode == "w" else tu).append(e0.elapsed_time(e1) * 1e3)
        over[f"{key[0]}-{key[1]}"] = round((float(np.median(tw)) / float(np.median(tu)) - 1) * 100, 2)
    rt.close()
    rt_m.close()
    t_alone = _agree_t_alone(t_alone, world, torch)
    n_total = args.scale_kernels
    mean_alone = float(np.mean([t_alone[(j["type"], j["size_class"])] for j in gen.queue_trace(6, n_total, 1)]))
    gap = int(mean_alone / (args.rho * world))                # offered load rho per GPU
    full = gen.queue_trace(6, n_total, gap)
    mine = assign_jobs(full, lambda j: t_alone[(j["type"], j["size_class"])], world)[rank]
    overhead_ns = 20_000
    _run_trace(F, torch, local, F.POLICY_FIFO, mine[:8], inst, t_alone, overhead_ns, streams)   # warm-up
    res = {}
    with ClockSampler(physical_gpu_index(local)) as clk:
        for name, pol in (("FIFO", F.POLICY_FIFO), ("HPF", F.POLICY_HPF)):
            turn, dec, evl, lat = _run_trace(F, torch, local, pol, mine, inst, t_alone, overhead_ns, streams,
                                             want_lat=True)
            res[name] = {"turn": [int(t[0]) for t in turn], "alone": [int(t_alone[t[1]]) for t in turn],
                         "makespan_ns": int(max(t[4] for t in turn)) if turn else 0,
                         "preemptions": sum(1 for d in dec if d[1] == 2), "lat_us": lat,
                         "lat_keys": list(_run_trace.lat_keys)}
    rec = {"rank": rank, "kernels": len(mine), "res": res, "clocks": clk.summary(), "overhead_pct": over}
    allr = gather_objects(rec, world)
    out = None
    if rank == 0:
        per_gpu, agg = [], {}
        for name in ("FIFO", "HPF"):
            tt = [x for r in allr for x in r["res"][name]["turn"]]
            al = [x for r in allr for x in r["res"][name]["alone"]]
            mk = max(r["res"][name]["makespan_ns"] for r in allr)
            agg[name] = {"antt": round(M.antt(tt, al), 3), "stp": round(M.stp(tt, al), 3),
                         "makespan_ms": round(mk / 1e6, 3),
                         "throughput_kernels_per_s": round(len(tt) / (mk / 1e9), 1) if mk else None}
        for r in allr:
            lat = r["res"]["HPF"]["lat_us"]
            per_gpu.append({"rank": r["rank"], "kernels": r["kernels"], "preemptions": r["res"]["HPF"]["preemptions"],
                            "preempt_latency_us": ({"p50": round(float(np.median(lat)), 2),
                                                    "p99": round(float(np.percentile(lat, 99)), 2),
                                                    "max": round(float(np.max(lat)), 2), "n": len(lat)} if lat else None),
                            "antt_hpf": round(M.antt(r["res"]["HPF"]["turn"], r["res"]["HPF"]["alone"]), 3) if r["kernels"] else None,
                            "antt_fifo": round(M.antt(r["res"]["FIFO"]["turn"], r["res"]["FIFO"]["alone"]), 3) if r["kernels"] else None,
                            "clocks": r["clocks"]})
        all_lat = [x for r in allr for x in r["res"]["HPF"]["lat_us"]]
        by_kernel = {}                 # the latency distribution per victim kernel (type-size class)
        for r in allr:
            for x, k in zip(r["res"]["HPF"]["lat_us"], r["res"]["HPF"].get("lat_keys", [])):
                by_kernel.setdefault(k, []).append(x)
        by_kernel = {k: {"p50": round(float(np.median(v)), 2), "max": round(float(np.max(v)), 2), "n": len(v)}
                     for k, v in sorted(by_kernel.items())}
        gain = agg["FIFO"]["antt"] / agg["HPF"]["antt"]
        out = {"metric": METRIC, "value": round(gain, 3), "unit": "x (ANTT_FIFO / ANTT_FLEP)",
               "value_definition": "NATT gain of FLEP-HPF over FIFO over all kernels of the shared job queue",
               "n_gpus": world, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
               "dtype": "mixed (f32, bf16->f32)", "data": "synthetic (seeded)",
               "config": {"workload": f"configs[4]: one job queue of {n_total} mixed kernels (seed 6) over {world} "
                                      f"independent per-GPU FLEP schedulers, Poisson arrivals at rho={args.rho} per GPU",
                          "mean_gap_us": round(gap / 1e3, 2), "parallelism": f"replicas x{world} (no collective on the path)",
                          "assignment": "least predicted backlog (sum of T_e), ties to the lowest rank"},
               "aggregate": agg, "per_gpu": per_gpu,
               "preempt_latency_us_all": ({"p50": round(float(np.median(all_lat)), 2),
                                           "p99": round(float(np.percentile(all_lat, 99)), 2),
                                           "max": round(float(np.max(all_lat)), 2), "n": len(all_lat)} if all_lat else None),
               "preempt_latency_us_by_victim": by_kernel,
               "wrapper_overhead_pct_rank0": allr[0]["overhead_pct"],
               "wrapper_overhead_pct_max_over_gpus": {k: max(r["overhead_pct"][k] for r in allr)
                                                      for k in allr[0]["overhead_pct"]}}
        _emit(out, rank, args)
    barrier(world)
    return out


# ------------------------------------------------------------------------------------------
def run_spatial_managed(args, rank, world, local):
    """configs[2] through the managed API (spatial HPF, R29): the runtime itself decides
    how far to preempt. A low-priority stencil5 fp32 16384^2 victim runs; a high-priority SAXPY-f32
    of n * k_wait blocks arrives (flep_launch, host) about 80 us later; the policy issues
    PREEMPT(victim, n) (n = ceil(workers / k), A9), launches the waiting kernel beside the victim
    and REFILLs the victim when it ends. n = 148 (the waiting kernel needs every SM) gives the
    temporal reference through the same path. Checked every trial: the decision list, I3 on the
    victim's first-epoch worker log (yield exits exactly on the SMs with rank < n), and the victim's
    output on sampled rows against a NumPy fp64 reference (bench_check)."""
    import torch
    import bench_check as BC
    from bench import ClockSampler, L2Flush, barrier, physical_gpu_index
    from paper_conf_asplos_wulzj17_b200 import flep as F
    torch.cuda.set_device(local)
    n_st = 16384
    g = torch.Generator(device="cuda")
    g.manual_seed(4 + rank)
    v_in = torch.rand(n_st, n_st, device="cuda", generator=g)
    v_out = torch.empty_like(v_in)
    rt = F.Runtime(device=local, policy=F.POLICY_HPF, spatial=True, keep_logs=True)
    k_v = rt.register_kernel(F.BODY_STENCIL5_F32, chunk=1, poll=1, name="victim", started_hint=True,
                             model=(0, 0, 0, 0, 330_000))
    k_w = rt.register_kernel(F.BODY_SAXPY_F32, chunk=1, poll=1, name="waiting", model=(0, 0, 0, 0, 10_000))
    cps_w, _ = rt.workers_for(F.BODY_SAXPY_F32)
    widths = [8, 16, 32, 74, rt.num_sms]
    wx = torch.rand(rt.num_sms * cps_w * 256, device="cuda", generator=g)
    wy = torch.rand(rt.num_sms * cps_w * 256, device="cuda", generator=g)
    flush = L2Flush(torch)
    A = torch.cuda.Stream(priority=0)
    B = torch.cuda.Stream(priority=-2)
    v_args, v_grid = F.stencil_args(v_out, v_in), F.stencil_grid(n_st)
    rng = gen.rng(2100 + rank)
    check_rows = sorted(set(int(r) for r in rng.integers(1, n_st - 1, 6)))
    slabs = {r: v_in[r - 1:r + 2].cpu().numpy() for r in check_rows}

    def spans(h):
        info = rt.query(h)
        evs = []
        for e_ in range(1, info.epoch + 1):
            evs += list(rt.events(h, e_))
        return _span(evs), info

    rows = []
    alone = {}
    with ClockSampler(physical_gpu_index(local)) as clk:
        # standalone times through the same runtime (nothing else queued: LAUNCH at once)
        for key, (k, grid, a) in {"victim": (k_v, v_grid, v_args)}.items():
            ts = []
            for r in range(3):
                flush.zero_()
                torch.cuda.synchronize()
                h = rt.launch(k, grid, a, stream=A)
                rt.sync(h)
                (t0, t1), _ = spans(h)
                if r:
                    ts.append((t1 - t0) / 1e3)
            alone[key] = float(np.median(ts))
        for n in widths:
            elems = n * cps_w * 256
            wa, wg = F.saxpy_f32_args(wy[:elems], wx[:elems], 0.5), F.saxpy_grid(elems)
            ts = []
            for r in range(3):
                flush.zero_()
                torch.cuda.synchronize()
                h = rt.launch(k_w, wg, wa, stream=B)
                rt.sync(h)
                (t0, t1), _ = spans(h)
                if r:
                    ts.append((t1 - t0) / 1e3)
            t_w = float(np.median(ts))
            lat, wstart, tflep, viol, bad_dec, worst, ok, mism = [], [], [], 0, 0, 0.0, 0, []
            for trial in range(args.warmup + args.steps):
                flush.zero_()
                torch.cuda.synchronize()
                nd0 = len(rt.decision_log())
                h_v = rt.launch(k_v, v_grid, v_args, priority=0, stream=A)
                t_w0 = time.perf_counter()
                while rt.query(h_v).started_epoch < 1 and time.perf_counter() - t_w0 < 1.0:
                    pass
                t_seen = F.now_ns()
                while F.now_ns() < t_seen + 80_000:
                    pass
                h_w = rt.launch(k_w, wg, wa, priority=1, stream=B)
                rt.sync(h_w, timeout_ns=10_000_000_000)
                rt.sync(h_v, timeout_ns=10_000_000_000)
                if trial < args.warmup:
                    continue
                dec = rt.decision_log()[nd0:]
                names = [(F.ACTION_NAMES[d[1]], d[2], d[3]) for d in dec]
                if n < rt.num_sms:
                    want = [("LAUNCH", h_v, 0), ("PREEMPT", h_v, n), ("LAUNCH", h_w, 0), ("REFILL", h_v, rt.num_sms)]
                else:
                    want = [("LAUNCH", h_v, 0), ("PREEMPT", h_v, rt.num_sms), ("LAUNCH", h_w, 0), ("RESUME", h_v, 0)]
                if names != want:
                    bad_dec += 1
                    if len(mism) < 3:
                        (v0_, v1_), iv = spans(h_v)
                        (w0_, w1_), iw = spans(h_w)
                        mism.append({"got": [(a_, int(i_ == h_v), int(n_)) for a_, i_, n_ in names],
                                     "want": [(a_, int(i_ == h_v), int(n_)) for a_, i_, n_ in want],
                                     "dev_us_from_victim_start": {"guest_start": (w0_ - v0_) / 1e3, "guest_end": (w1_ - v0_) / 1e3,
                                                                  "victim_end": (v1_ - v0_) / 1e3},
                                     "host_us_from_victim_arrive": {"guest_arrive": (iw.t_arrive - iv.t_arrive) / 1e3,
                                                                    "guest_finish": (iw.t_finish - iv.t_arrive) / 1e3,
                                                                    "victim_finish": (iv.t_finish - iv.t_arrive) / 1e3,
                                                                    "guest_first_start": (iw.t_first_start - iv.t_arrive) / 1e3},
                                     "victim_epochs": iv.epoch, "guest_workers": iw.workers})
                    continue
                info_v = rt.query(h_v)
                ev1 = rt.events(h_v, 1)
                (v0, v1), _ = spans(h_v)
                (w0, w1), _ = spans(h_w)
                if n < rt.num_sms:
                    # I3: the workers on the n released SMs (rank = smid) yield; no other worker
                    # leaves before the waiting kernel is done (the REFILL then widens the request
                    # to every SM, so later yields elsewhere are the refill's)
                    viol += sum(1 for e in ev1 if e.smid < n and e.reason != F.REASON_YIELD)
                    viol += sum(1 for e in ev1 if e.smid >= n and e.reason == F.REASON_YIELD and e.t_exit < w1)
                off = t_seen - v0                                 # host - device (started hint)
                # the PREEMPT decision's host time (the runtime writes the request right after it;
                # t_last_request is overwritten by the REFILL's request)
                t_pre = [d[0] for d in dec if d[1] == 2 and d[2] == h_v]
                t_req = t_pre[0] - off if t_pre else None
                ys = [e.t_exit for e in ev1 if e.reason == F.REASON_YIELD]
                if ys and t_req:
                    lat.append((max(ys) - t_req) / 1e3)
                if t_req:
                    wstart.append((w0 - t_req) / 1e3)
                tflep.append((max(v1, w1) - v0) / 1e3)
                ok += 1
            got = {r: v_out[r].cpu().numpy() for r in check_rows}
            for r in check_rows:
                ref, den = BC.stencil5_f32(slabs[r])
                d = np.maximum(np.abs(ref[1]), den[1])
                worst = max(worst, float(np.max(np.abs(got[r] - ref[1]) / np.where(d > 0, d, 1))))
            t_org = alone["victim"] + t_w
            rows.append({"n_sms": n, "trials": ok, "decision_list_mismatches": bad_dec, "I3_violations": viol,
                         "mismatch_examples": mism,
                         "yield_latency_us_p50": round(float(np.median(lat)), 3) if lat else None,
                         "waiting_start_us_p50": round(float(np.median(wstart)), 3) if wstart else None,
                         "t_flep_us": round(float(np.median(tflep)), 2) if tflep else None,
                         "t_org_us": round(t_org, 2), "t_waiting_alone_us": round(t_w, 2),
                         "overhead": round((float(np.median(tflep)) - t_org) / t_org, 4) if tflep else None,
                         "victim_rows_max_rel": worst, "victim_parity_ok": bool(worst <= 1e-5)})
    temporal = rows[-1]
    for r in rows:
        r["overhead_reduction_vs_temporal"] = (round(1.0 - r["overhead"] / temporal["overhead"], 4)
                                               if r["overhead"] is not None and temporal["overhead"] else None)
    dec_all = rt.decision_log()
    evl = rt.event_log_ex()
    rt.close()
    import os
    ev_dir = os.environ.get("FLEP_EVIDENCE_DIR")
    if ev_dir and rank == 0:
        with open(os.path.join(ev_dir, "spatial_managed_logs.json"), "w") as fh:
            json.dump({"workload": "configs[2] managed spatial HPF", "num_sms": 148,
                       "events": [list(map(int, e)) for e in evl], "decisions": [list(map(int, d)) for d in dec_all]}, fh)
    out = {"metric": METRIC, "value": rows[0]["overhead_reduction_vs_temporal"],
           "unit": "fraction (1 - ovh_spatial / ovh_temporal)",
           "value_definition": "managed spatial HPF: preemption-overhead reduction of the runtime's 8-SM decision vs "
                               "its temporal decision for a waiting kernel that needs every SM (P:297, Fig. 15)",
           "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "higher_is_better": True,
           "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic (seeded)",
           "config": {"workload": "configs[2] via the managed API: stencil5 fp32 16384^2 victim (prio 0) + SAXPY-f32 "
                                  "of n*k_wait blocks (prio 1), n in {8,16,32,74,148}; HPF with spatial decisions",
                      "l2": "flushed between trials", "victim_chunk": 1, "poll": 1},
           "t_victim_alone_us": round(alone["victim"], 2), "per_width": rows,
           "decisions_ok": all(r["decision_list_mismatches"] == 0 for r in rows),
           "I3_violations": sum(r["I3_violations"] for r in rows),
           "victim_parity_ok": all(r["victim_parity_ok"] for r in rows),
           "clocks": clk.summary()}
    _emit(out, rank, args)
    barrier(world)
    return out


# ------------------------------------------------------------------------------------------
def run_slicing_overhead(args, rank, world, local):
    """E13 (Fig. 17): overhead of the preemption mechanisms when NOTHING preempts,
    per kernel, against the unwrapped grid: FLEP's persistent workers (the queue's tuned C and the
    latency setting C = 1), kernel slicing with every slice enqueued and the device check at slice
    entry (R31; slice = one wave W*C*K, A20), and plain back-to-back slices without any check (the
    lower bound of slicing: launch gaps only). CUDA events on the launching stream, dithered, L2
    flushed, interleaved; trimmed mean of `reps` samples."""
    import torch
    from bench import ClockSampler, L2Flush, barrier, physical_gpu_index
    from paper_conf_asplos_wulzj17_b200 import flep as F
    from paper_conf_asplos_wulzj17_b200.calibrate import dither, event_mean_us
    torch.cuda.set_device(local)
    inst = _queue_instances(torch, F, seed=5)
    flush = L2Flush(torch)
    S = torch.cuda.Stream()
    rt_m = F.Runtime(device=local, exec_on_user_stream=True)
    rt_s = F.Runtime(device=local, policy=F.POLICY_SLICE_DEVICE, exec_on_user_stream=True)
    rows = []
    reps = max(8, args.reps // 4)
    with ClockSampler(physical_gpu_index(local)) as clk:
        for key in sorted(inst):
            body, grid, a, keep, _ = inst[key]
            C = _qopts(F, key[0], body)["chunk"]
            k_t = rt_m.register_kernel(body, **_qopts(F, key[0], body))
            k_1 = rt_m.register_kernel(body, chunk=1, poll=1, in_tile=body in (F.BODY_GEMM_BF16, F.BODY_GEMM_BF16_2SM, F.BODY_GEMM_BF16_2SM_W))
            k_s = rt_s.register_kernel(body, chunk=C, poll=1)
            cps, w = rt_m.workers_for(body)
            slice_blocks = w * C                                     # one wave of W*C*K blocks (A20)
            t = {m: [] for m in ("unwrapped", "static_u1", "flep_tuned", "flep_c1", "slice_device", "slice_plain")}
            for r in range(reps + 2):
                for m in t:
                    with torch.cuda.stream(S):
                        flush.zero_()
                        dither(torch)
                        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                        e0.record(S)
                    h = None
                    if m == "unwrapped":
                        rt_m.launch_unwrapped(body, grid, a, stream=S)
                    elif m == "static_u1":
                        rt_m.launch_static(body, grid, a, chunk=C, stream=S)
                    elif m == "flep_tuned":
                        h = (rt_m, rt_m.launch(k_t, grid, a, stream=S))
                    elif m == "flep_c1":
                        h = (rt_m, rt_m.launch(k_1, grid, a, stream=S))
                    elif m == "slice_device":
                        h = (rt_s, rt_s.launch(k_s, grid, a, stream=S))
                    else:
                        rt_m.launch_sliced(body, grid, a, slice_blocks, stream=S)
                    e1.record(S)
                    e1.synchronize()
                    if h is not None:
                        h[0].sync(h[1])
                    if r >= 2:
                        t[m].append(e0.elapsed_time(e1) * 1e3)
            u = event_mean_us(t["unwrapped"])
            nb = grid[0] * grid[1]
            row = {"kernel": f"{key[0]}-{key[1]}", "blocks": nb, "slice_blocks": slice_blocks,
                   "slices": -(-nb // slice_blocks), "unwrapped_us": round(u, 2)}
            for m in ("static_u1", "flep_tuned", "flep_c1", "slice_device", "slice_plain"):
                v = event_mean_us(t[m])
                row[m + "_us"] = round(v, 2)
                row[m + "_overhead_pct"] = round((v / u - 1) * 100, 2)
            row["flep_tuned_over_static_pct"] = round((row["flep_tuned_us"] / row["static_u1_us"] - 1) * 100, 2)
            row["tuned_chunk"] = C
            rows.append(row)
        # the CTA-pair GEMM (R32) at the largest size: cuBLAS, unwrapped, U1 and the FLEP pair
        # workers, interleaved
        A8, B8, C8 = inst[("gemm_bf16", 2)][3]
        a8 = F.gemm_args(C8, A8, B8)
        g2 = F.gemm2_grid(C8.shape[0], C8.shape[1])
        k2 = {c: rt_m.register_kernel(F.BODY_GEMM_BF16_2SM, chunk=c, poll=1) for c in (1, 2)}
        g2w = F.gemm2w_grid(C8.shape[0], C8.shape[1])          # the 256x512 pair tile
        k2w = rt_m.register_kernel(F.BODY_GEMM_BF16_2SM_W, chunk=1, poll=1)
        tg = {m: [] for m in ("cublas", "unwrapped", "static_u1", "flep_c1", "flep_c2",
                              "wide_unwrapped", "wide_static_u1", "wide_flep_c1")}
        for r in range(max(6, reps // 2) + 2):
            for m in tg:
                with torch.cuda.stream(S):
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(S)
                    h = None
                    if m == "cublas":
                        torch.matmul(A8, B8.t(), out=C8)
                    elif m == "unwrapped":
                        rt_m.launch_unwrapped(F.BODY_GEMM_BF16_2SM, g2, a8, stream=S)
                    elif m == "static_u1":
                        rt_m.launch_static(F.BODY_GEMM_BF16_2SM, g2, a8, stream=S)
                    elif m == "wide_unwrapped":
                        rt_m.launch_unwrapped(F.BODY_GEMM_BF16_2SM_W, g2w, a8, stream=S)
                    elif m == "wide_static_u1":
                        rt_m.launch_static(F.BODY_GEMM_BF16_2SM_W, g2w, a8, stream=S)
                    elif m == "wide_flep_c1":
                        h = rt_m.launch(k2w, g2w, a8, stream=S)
                    else:
                        h = rt_m.launch(k2[1 if m == "flep_c1" else 2], g2, a8, stream=S)
                    e1.record(S)
                e1.synchronize()
                if h is not None:
                    rt_m.sync(h)
                if r >= 2:
                    tg[m].append(e0.elapsed_time(e1) * 1e3)
        gm = {m: float(np.median(v)) for m, v in tg.items()}
        flop = 2.0 * C8.shape[0] * C8.shape[1] * A8.shape[1]
        gemm2 = {"size": f"{C8.shape[0]}x{C8.shape[1]}x{A8.shape[1]} bf16", "stat": "median, interleaved",
                 **{m + "_us": round(v, 2) for m, v in gm.items()},
                 **{m + "_tflops": round(flop / v / 1e6, 1) for m, v in gm.items()},
                 "flep_c2_vs_cublas": round(gm["cublas"] / gm["flep_c2"], 3),
                 "flep_c2_over_static_pct": round((gm["flep_c2"] / gm["static_u1"] - 1) * 100, 2),
                 "flep_c1_over_static_pct": round((gm["flep_c1"] / gm["static_u1"] - 1) * 100, 2),
                 "wide_flep_c1_vs_cublas": round(gm["cublas"] / gm["wide_flep_c1"], 3),
                 "wide_flep_c1_over_static_pct": round((gm["wide_flep_c1"] / gm["wide_static_u1"] - 1) * 100, 2)}
        # the wrapped tensor-core kernel against the tensor roofline (burst peak: a kernel timed
        # alone between others, MEASURED_PEAKS.json)
        from bench import peaks
        _, pk_burst, pk_sus, pk_src = peaks()
        ach = flop / gm["wide_flep_c1"] / 1e6
        gemm2["roofline"] = {"bound": "tensor", "kernel": "flep_gemm2_worker<Gemm2T<512>> C = 1",
                             "achieved": round(ach, 1), "peak": pk_burst, "unit": "TFLOP/s",
                             "frac": round(ach / pk_burst, 4), "peak_source": pk_src + " (burst)",
                             "frac_of_sustained_peak": round(ach / pk_sus, 4)}
    rt_m.close()
    rt_s.close()
    big = [r for r in rows if r["kernel"].endswith("-2")]
    mean = lambda k, rs: round(float(np.mean([r[k] for r in rs])), 2)  # noqa: E731
    out = {"metric": METRIC, "value": mean("flep_tuned_overhead_pct", rows), "unit": "% over the unwrapped grid",
           "value_definition": "mean never-preempted overhead of FLEP (tuned C) over the 12 queue kernels (E13, Fig. 17)",
           "n_gpus": world, "higher_is_better": False, "scaling": "weak", "vs_baseline": None,
           "dtype": "mixed", "data": "synthetic (seeded)",
           "config": {"workload": "E13: the configs[3] queue's 12 kernel instances run alone, never preempted",
                      "reps": reps, "l2": "flushed between samples"},
           "mean_overhead_pct": {k: mean(k + "_overhead_pct", rows) for k in ("static_u1", "flep_tuned", "flep_c1", "slice_device", "slice_plain")},
           "mean_overhead_pct_large": {k: mean(k + "_overhead_pct", big) for k in ("static_u1", "flep_tuned", "flep_c1", "slice_device", "slice_plain")},
           "paper": "FLEP 2.5 % vs kernel slicing 8 % at the same preemption granularity (P:391, K40)",
           "kernels": rows, "gemm_2sm_8192": gemm2, "clocks": clk.summary()}
    _emit(out, rank, args)
    barrier(world)
    return out
