"""GPU tests of the request relay (FLEP_KFLAG_HOST_RELAY, R28): the extra relay CTA is
not a worker (W = k x SMs - 1, results and coverage unchanged), leaves with its epoch (no hang
under device-triggered or host-issued requests), and host requests still preempt exactly-once."""
import time

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


@pytest.mark.parametrize("n", [256, (1 << 20) + 3])
def test_relay_saxpy_exact(rt, n):
    f = flep_mod()
    x, y = gen.saxpy_i32_inputs(n, seed=71)
    k = rt.register_kernel(f.BODY_SAXPY_I32, chunk=2, poll=1, host_relay=True)
    xd, yd = t(x), t(y)
    h = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, 5))
    rt.sync(h, timeout_ns=10_000_000_000)
    nb = f.saxpy_grid(n)[0]
    assert np.all(rt.coverage_np(h, nb) == 1)
    assert np.array_equal(yd.cpu().numpy(), W.saxpy_i32(5, x, y))
    info = rt.query(h)
    _, wmax = rt.workers_for(f.BODY_SAXPY_I32)
    assert info.workers == min(wmax - 1, -(-nb // 2))


@pytest.mark.parametrize("seed", range(3))
def test_relay_device_triggered_schedules(rt, seed):
    f = flep_mod()
    n = 1 << 20
    nb = n // 256
    x, y = gen.saxpy_i32_inputs(n, seed=72 + seed)
    k = rt.register_kernel(f.BODY_SAXPY_I32, chunk=1, poll=1, host_relay=True)
    xd, yd = t(x), t(y)
    sched = gen.preempt_schedule(950 + seed, nb, rt.num_sms)
    h, npre, viol = run_manual_schedule(rt, k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, 3), nb, sched,
                                        rt.num_sms)
    assert viol == []
    assert np.all(rt.coverage_np(h, nb) == 1)
    assert np.array_equal(yd.cpu().numpy(), W.saxpy_i32(3, x, y))


def test_relay_host_request_preempts_and_resumes(rt):
    f = flep_mod()
    rows = 1 << 22
    rp, col, val, xv = gen.csr_inputs(rows, seed=73)
    import torch
    y = torch.zeros(rows, device="cuda")
    k = rt.register_kernel(f.BODY_SPMV_CSR_F32, chunk=1, poll=1, host_relay=True, started_hint=True)
    keep = (t(rp), t(col), t(val), t(xv))       # outlive the args struct (raw pointers)
    h = rt.launch(k, f.spmv_grid(rows), f.spmv_args(y, *keep))
    t0 = time.perf_counter()
    while rt.query(h).started_epoch < 1 and time.perf_counter() - t0 < 1:
        pass
    time.sleep(30e-6)
    try:
        rt.preempt(h, rt.num_sms)
    except f.FlepError:
        pass                                   # already complete
    rt.wait_epoch(h, timeout_ns=10_000_000_000)
    if rt.query(h).state == f.STATE_PREEMPTED:
        rt.resume(h)
    rt.sync(h, timeout_ns=10_000_000_000)
    nb = f.spmv_grid(rows)[0]
    assert np.all(rt.coverage_np(h, nb) == 1)
    ref, absum = W.spmv_csr(rp, col, val, xv)
    got = y.cpu().numpy().astype(np.float64)
    d = np.maximum(np.abs(ref), absum)
    assert float(np.max(np.abs(got - ref) / np.where(d > 0, d, 1.0))) <= 1e-5


@pytest.mark.parametrize("seed", range(6))
def test_relay_leaves_a_released_sm(rt, seed):
    """I3 for every CTA of the grid: a host spatial request of n SMs makes the relay
    CTA leave if its own SM is among the released ones (rank = smid < n), before the epoch ends;
    otherwise it stays until the epoch is published. Workers yield only on the released SMs."""
    f = flep_mod()
    import torch
    rows = 1 << 22
    rp, col, val, xv = gen.csr_inputs(rows, seed=74)
    y = torch.zeros(rows, device="cuda")
    k = rt.register_kernel(f.BODY_SPMV_CSR_F32, chunk=1, poll=1, host_relay=True, started_hint=True)
    g = gen.rng(4000 + seed)
    n = int(g.integers(1, rt.num_sms))
    keep = (t(rp), t(col), t(val), t(xv))       # outlive the args struct (raw pointers)
    h = rt.launch(k, f.spmv_grid(rows), f.spmv_args(y, *keep))
    t0 = time.perf_counter()
    while rt.query(h).started_epoch < 1 and time.perf_counter() - t0 < 1:
        pass
    try:
        rt.preempt(h, n)
    except f.FlepError:
        pytest.skip("the launch completed before the request")
    rt.sync(h, timeout_ns=10_000_000_000)           # spatial: the rest of the workers finish it
    ep = rt.epoch_info(h, 1)
    assert ep.relay_reason in (f.RELAY_LEFT_OWN_SM, f.RELAY_LEFT_PUBLISHED)
    if ep.relay_smid < n:
        assert ep.relay_reason == f.RELAY_LEFT_OWN_SM
        assert ep.relay_t_exit <= ep.t_end
    else:
        assert ep.relay_reason == f.RELAY_LEFT_PUBLISHED
    for e in rt.events(h, 1):
        if e.reason == f.REASON_YIELD:
            assert e.smid < n
    nb = f.spmv_grid(rows)[0]
    assert np.all(rt.coverage_np(h, nb) == 1)
