"""GPU tests of the speculative fetch (FLEP_KFLAG_SPEC_FETCH, R34): at a poll point the
task-fetch atomic and the poll load are in flight together; a worker that must leave returns the
chunk it fetched through its record, and the worker with the same index runs it first in the next
epoch. Checked: every block exactly once under random preempt/resume schedules (temporal and
spatial, I3), outputs bit-identical to uninterrupted runs and to the oracle, a yielding worker runs
nothing after the request (its fetched chunk is returned whole), and the flag's exclusions."""
import numpy as np
import pytest

from oracle import workloads as W
from synth import gen

from flep_gpu_util import flep_mod, run_manual_schedule, t

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def rt():
    f = flep_mod()
    r = f.Runtime(coverage=True)
    yield r
    r.close()


def test_spec_fetch_random_schedules_saxpy(rt):
    f = flep_mod()
    n, a = 1 << 20, 1664525
    nb = n // 256
    x, y = gen.saxpy_i32_inputs(n, seed=11)
    ref = W.saxpy_i32(a, x, y)
    xd, y0, yd = t(x), t(y), t(y)
    kern, bad = {}, []
    for i in range(600):
        s = gen.preempt_schedule(7000 + i, nb, rt.num_sms)
        key = (s["C"], s["K"], i % 3)
        if key not in kern:
            kern[key] = rt.register_kernel(f.BODY_SAXPY_I32, chunk=s["C"], poll=s["K"], spec_fetch=True,
                                           ctas_per_sm=(1, 2, 8)[i % 3])
        yd.copy_(y0)
        h, npre, viol = run_manual_schedule(rt, kern[key], f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, a), nb,
                                            s, rt.num_sms, check_prefix=False)
        if not np.all(rt.coverage_np(h, nb) == 1):
            viol.append("I1: coverage != 1")
        if i % 10 == 0 and not np.array_equal(yd.cpu().numpy(), ref):
            viol.append("result != oracle")
        if viol:
            bad.append((i, s, viol))
    assert not bad, bad[:3]


@pytest.mark.parametrize("body", ["spmv", "spmv_vec", "stencil", "stencil_tma"])
def test_spec_fetch_preempt_resume_bitexact(rt, body):
    import torch
    f = flep_mod()
    if body.startswith("spmv"):
        rows = (1 << 18) + 19
        rowptr, col, val, x = gen.csr_inputs(rows, seed=51)
        keep = (t(rowptr), t(col), t(val), t(x))
        out = torch.zeros(rows, device="cuda")
        bid = f.BODY_SPMV_CSR_F32 if body == "spmv" else f.BODY_SPMV_CSR_F32_VEC
        grid, args = f.spmv_grid(rows), f.spmv_args(out, *keep)
    else:
        a = gen.stencil_f32_input(2048, seed=52)
        ind = t(a)
        out = torch.zeros_like(ind)
        bid = f.BODY_STENCIL5_F32 if body == "stencil" else f.BODY_STENCIL5_F32_TMA
        grid, args = f.stencil_grid(2048), f.stencil_args(out, ind)
    nb = grid[0] * grid[1]
    rt.launch_unwrapped(bid, grid, args)
    torch.cuda.synchronize()
    base = out.clone()
    for C, K in ((1, 1), (1, 3), (2, 1), (4, 2)):
        k = rt.register_kernel(bid, chunk=C, poll=K, spec_fetch=True)
        for cyc in range(4):
            out.zero_()
            sched = gen.preempt_schedule(8000 + 10 * C + cyc, nb, rt.num_sms)
            h, npre, viol = run_manual_schedule(rt, k, grid, args, nb, sched, rt.num_sms, check_prefix=False)
            assert viol == []
            assert np.all(rt.coverage_np(h, nb) == 1)
            assert torch.equal(out, base)
    if body.startswith("spmv"):
        ref, absum = W.spmv_csr(rowptr, col, val, x)
        got = base.cpu().numpy().astype(np.float64)
        d = np.maximum(np.abs(ref), absum)
        assert float(np.max(np.abs(got - ref) / np.where(d > 0, d, 1))) <= 1e-5


def test_spec_fetch_returns_whole_chunks(rt):
    """C = 8, temporal request: the drained epoch ran the counter's blocks except the returned
    chunks; each hole is a whole fetched chunk [b, b + 8) (nothing of it ran), at most one per
    yielding worker; the resume runs them exactly once."""
    f = flep_mod()
    n = 1 << 24
    nb = n // 256
    C = 8
    x, y = gen.saxpy_i32_inputs(n, seed=53)
    xd, yd = t(x), t(y)
    k = rt.register_kernel(f.BODY_SAXPY_I32, chunk=C, poll=1, spec_fetch=True)
    rt.arm_next_trigger(nb // 2, rt.num_sms)
    h = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, 3))
    rt.wait_epoch(h, timeout_ns=10_000_000_000)
    info = rt.query(h)
    assert info.state == f.STATE_PREEMPTED
    cov = rt.coverage_np(h, nb)
    ctr = min(int(info.counter), nb)
    assert np.all(cov[ctr:] == 0) and np.all(cov <= 1)
    assert info.blocks_done == int(cov.sum())
    holes = np.flatnonzero(cov[:ctr] == 0)
    assert holes.size > 0                               # fetched chunks were returned, not run
    starts = holes[(holes % C) == 0]
    assert holes.size == C * starts.size                # whole chunks, aligned like the fetch
    assert np.all(np.isin(holes, (starts[:, None] + np.arange(C)).ravel()))
    ys = [e for e in rt.events(h, 1) if e.reason == f.REASON_YIELD]
    assert starts.size <= len(ys)
    rt.resume(h)
    rt.sync(h, timeout_ns=10_000_000_000)
    assert np.all(rt.coverage_np(h, nb) == 1)
    assert np.array_equal(yd.cpu().numpy(), W.saxpy_i32(3, x, y))


def test_spec_fetch_exclusions(rt):
    f = flep_mod()
    for kw in ({"prefetch": True}, {"async_poll": True}, {"clc": True}, {"sched_warp": True},
               {"warp_tasks": True}):
        with pytest.raises(f.FlepError):
            rt.register_kernel(f.BODY_SAXPY_I32, chunk=1, poll=1, spec_fetch=True, **kw)
    with pytest.raises(f.FlepError):
        rt.register_kernel(f.BODY_GEMM_BF16, chunk=1, poll=1, spec_fetch=True)
