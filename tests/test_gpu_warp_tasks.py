"""GPU tests of the warp-task worker (FLEP_KFLAG_WARP_TASKS, R30): a task is one warp's
share of an original block and every warp of a worker CTA fetches, polls and exits on its own.

Checked against the oracle and against the other forms of the same body: every task exactly once
(coverage counted per task), preempted epochs cover a task prefix (I2), yields only on the
requested SMs (I3), outputs bit-identical to the unwrapped grid and to uninterrupted runs, and
within the fp32 tolerance of the oracle."""
import numpy as np
import pytest

from oracle import workloads as W
from synth import gen

from flep_gpu_util import flep_mod, run_manual_schedule, t

pytestmark = pytest.mark.gpu

REL_FP32 = 1e-5
TPB = 8


@pytest.fixture(scope="module")
def torch_mod():
    import torch
    return torch


@pytest.fixture(scope="module")
def rt():
    f = flep_mod()
    r = f.Runtime(coverage=True)
    yield r
    r.close()


def _rel_err(got, ref, denom):
    d = np.maximum(np.abs(ref), denom)
    d = np.where(d > 0, d, 1.0)
    return float(np.max(np.abs(got.astype(np.float64) - ref) / d)) if got.size else 0.0


@pytest.mark.parametrize("rows,runs", [(1, []), (33, []), (5000, []), (6000, [(0, 300), (1000, 1800), (5600, 6000)]),
                                       ((1 << 16) + 5, [])])
def test_spmv_vec_all_forms_agree(rt, torch_mod, rows, runs):
    f = flep_mod()
    rowptr, col, val, x = gen.csr_inputs(rows, seed=31, empty_runs=runs)
    ref, absum = W.spmv_csr(rowptr, col, val, x)
    dr, dc, dv, dx = t(rowptr), t(col), t(val), t(x)
    grid = f.spmv_grid(rows)
    nb = grid[0]
    outs = {}
    yu = torch_mod.full((rows,), float("nan"), device="cuda")
    rt.launch_unwrapped(f.BODY_SPMV_CSR_F32_VEC, grid, f.spmv_args(yu, dr, dc, dv, dx))
    torch_mod.cuda.synchronize()
    outs["unwrapped"] = yu.cpu().numpy()
    for name, kw in (("counter", dict(chunk=1)), ("warp1", dict(chunk=1, warp_tasks=True)),
                     ("warp3", dict(chunk=3, warp_tasks=True)), ("warp8pf", dict(chunk=8, warp_tasks=True, prefetch=True)),
                     ("clc", dict(chunk=2, clc=True))):
        k = rt.register_kernel(f.BODY_SPMV_CSR_F32_VEC, poll=1, **kw)
        yd = torch_mod.full((rows,), float("nan"), device="cuda")
        h = rt.launch(k, grid, f.spmv_args(yd, dr, dc, dv, dx))
        rt.sync(h)
        outs[name] = yd.cpu().numpy()
        info = rt.query(h)
        per = TPB if kw.get("warp_tasks") else 1
        assert info.tasks_per_block == per
        assert info.blocks_total == nb * per
        assert np.all(rt.coverage_np(h, nb * per) == 1), name
    assert _rel_err(outs["unwrapped"], ref, absum) <= REL_FP32
    for name, y in outs.items():
        assert np.array_equal(y, outs["unwrapped"]), name      # same per-row arithmetic everywhere


@pytest.mark.parametrize("n", [64, 130, 1000, 4096])
@pytest.mark.parametrize("integer", [False, True])
def test_stencil_warp_tasks_bitexact(rt, torch_mod, n, integer):
    f = flep_mod()
    body = f.BODY_STENCIL5_I32 if integer else f.BODY_STENCIL5_F32
    a = gen.stencil_i32_input(n, seed=32) if integer else gen.stencil_f32_input(n, seed=32)
    ind = t(a)
    k = rt.register_kernel(body, chunk=2, poll=1, warp_tasks=True)
    outd = torch_mod.empty_like(ind)
    h = rt.launch(k, f.stencil_grid(n), f.stencil_args(outd, ind))
    rt.sync(h)
    got = outd.cpu().numpy()
    nb = f.stencil_grid(n)[0] * f.stencil_grid(n)[1]
    assert np.all(rt.coverage_np(h, nb * TPB) == 1)
    if integer:
        assert np.array_equal(got, W.stencil5_i32(a))
    else:
        ref, absum = W.stencil5_f32(a)
        assert _rel_err(got, ref, absum) <= REL_FP32
    out2 = torch_mod.empty_like(ind)
    rt.launch_unwrapped(body, f.stencil_grid(n), f.stencil_args(out2, ind))
    torch_mod.cuda.synchronize()
    assert np.array_equal(out2.cpu().numpy(), got)


@pytest.mark.parametrize("which", ["spmv", "stencil_i32"])
def test_warp_task_schedules_exactly_once(rt, torch_mod, which):
    """300 random manual preempt/resume schedules (temporal and spatial, device triggers at random
    blocks, C in {1,2,4,8,16} tasks, K in {1,2,4,8}, with and without prefetch / async poll):
    every task exactly once, preempted epochs cover a task prefix, yields only on requested SMs,
    output identical to the uninterrupted run."""
    f = flep_mod()
    if which == "spmv":
        rows = (1 << 16) + 77
        rowptr, col, val, x = gen.csr_inputs(rows, seed=33)
        dr, dc, dv, dx = t(rowptr), t(col), t(val), t(x)
        body, grid = f.BODY_SPMV_CSR_F32_VEC, f.spmv_grid(rows)
        out = torch_mod.zeros(rows, device="cuda")
        args = f.spmv_args(out, dr, dc, dv, dx)
        ref_fn = lambda: W.spmv_csr(rowptr, col, val, x)  # noqa: E731
    else:
        n = 1000
        a = gen.stencil_i32_input(n, seed=34)
        ind = t(a)
        out = torch_mod.zeros_like(ind)
        body, grid = f.BODY_STENCIL5_I32, f.stencil_grid(n)
        args = f.stencil_args(out, ind)
        ref_fn = lambda: W.stencil5_i32(a)  # noqa: E731
    nb = grid[0] * grid[1]
    k0 = rt.register_kernel(body, chunk=4, warp_tasks=True)
    h0 = rt.launch(k0, grid, args)
    rt.sync(h0)
    base = out.clone()
    kern, viol_all = {}, []
    for i in range(300):
        s = gen.preempt_schedule(900 + i, nb, rt.num_sms)
        pf, ap = i % 2 == 1, (i // 2) % 2 == 1
        key = (s["C"], s["K"], pf, ap)
        if key not in kern:
            kern[key] = rt.register_kernel(body, chunk=s["C"], poll=s["K"], prefetch=pf, async_poll=ap,
                                           warp_tasks=True)
        out.zero_()
        h, npre, viol = run_manual_schedule(rt, kern[key], grid, args, nb * TPB, s, rt.num_sms,
                                            check_prefix=(i % 5 == 0))
        if not np.all(rt.coverage_np(h, nb * TPB) == 1):
            viol.append("I1: task coverage != 1")
        if not torch_mod.equal(out, base):
            viol.append("output differs from the uninterrupted run")
        if viol:
            viol_all.append((i, s, viol))
    assert not viol_all, viol_all[:3]
    got = base.cpu().numpy()
    if which == "spmv":
        ref, absum = ref_fn()
        assert _rel_err(got, ref, absum) <= REL_FP32
    else:
        assert np.array_equal(got, ref_fn())


def test_warp_task_temporal_drain_and_worker_log(rt, torch_mod):
    """A temporal request reaches every warp worker: the drained epoch's worker log has one
    record per warp (W = CTAs x 8), all of them yields or exhausted, on real SMs."""
    f = flep_mod()
    rows = 1 << 20
    rowptr, col, val, x = gen.csr_inputs(rows, seed=2)
    dr, dc, dv, dx = t(rowptr), t(col), t(val), t(x)
    yd = torch_mod.zeros(rows, device="cuda")
    k = rt.register_kernel(f.BODY_SPMV_CSR_F32_VEC, chunk=1, poll=1, warp_tasks=True)
    grid = f.spmv_grid(rows)
    rt.arm_next_trigger(grid[0] // 2, rt.num_sms)
    h = rt.launch(k, grid, f.spmv_args(yd, dr, dc, dv, dx))
    rt.wait_epoch(h, timeout_ns=10_000_000_000)
    info = rt.query(h)
    assert info.state == f.STATE_PREEMPTED
    ev = rt.events(h, 1)
    assert len(ev) == info.workers and info.workers % TPB == 0
    assert sum(1 for e in ev if e.reason == f.REASON_YIELD) > info.workers // 2
    ep = rt.epoch_info(h, 1)
    assert ep.trigger_block == (grid[0] // 2) * TPB
    rt.resume(h)
    rt.sync(h)
    assert np.all(rt.coverage_np(h, grid[0] * TPB) == 1)
    ref, absum = W.spmv_csr(rowptr, col, val, x)
    assert _rel_err(yd.cpu().numpy(), ref, absum) <= REL_FP32
