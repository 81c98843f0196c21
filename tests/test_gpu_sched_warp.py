"""GPU parity of the scheduling-warp worker (FLEP_KFLAG_SCHED_WARP, R26): same results as
the oracle and as the plain worker (bit for bit: the bodies are unchanged), coverage == 1, and the
preemption protocol (temporal and spatial requests, resume) exactly-once with drained epochs that
cover a counter prefix (I2)."""
import numpy as np
import pytest

from oracle import workloads as W
from synth import gen

from flep_gpu_util import flep_mod, run_manual_schedule, t

pytestmark = pytest.mark.gpu


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


@pytest.mark.parametrize("n", [1, 4099, (1 << 20) + 3])
@pytest.mark.parametrize("chunk,poll", [(1, 1), (8, 2)])
def test_sw_saxpy_exact(rt, torch_mod, n, chunk, poll):
    f = flep_mod()
    x, y = gen.saxpy_i32_inputs(n, seed=51)
    k = rt.register_kernel(f.BODY_SAXPY_I32, chunk=chunk, poll=poll, sched_warp=True)
    xd, yd = t(x), t(y)
    h = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, 1664525))
    rt.sync(h, timeout_ns=10_000_000_000)
    nb = f.saxpy_grid(n)[0]
    assert np.all(rt.coverage_np(h, nb) == 1)
    assert np.array_equal(yd.cpu().numpy(), W.saxpy_i32(1664525, x, y))
    info = rt.query(h)
    assert info.state == f.STATE_DONE and info.counter == -(-nb // chunk) * chunk + info.workers * chunk


def test_sw_spmv_bitwise_equal_to_plain_worker(rt, torch_mod):
    f = flep_mod()
    rows = (1 << 16) + 77
    rp, col, val, x = gen.csr_inputs(rows, seed=52)
    args_in = (t(rp), t(col), t(val), t(x))
    y0 = torch_mod.zeros(rows, device="cuda")
    y1 = torch_mod.zeros(rows, device="cuda")
    for sw, y in ((False, y0), (True, y1)):
        k = rt.register_kernel(f.BODY_SPMV_CSR_F32, chunk=1, poll=1, sched_warp=sw)
        h = rt.launch(k, f.spmv_grid(rows), f.spmv_args(y, *args_in))
        rt.sync(h, timeout_ns=10_000_000_000)
        assert np.all(rt.coverage_np(h, f.spmv_grid(rows)[0]) == 1)
    assert torch_mod.equal(y0.view(torch_mod.int32), y1.view(torch_mod.int32))
    ref, absum = W.spmv_csr(rp, col, val, x)
    got = y1.cpu().numpy().astype(np.float64)
    d = np.maximum(np.abs(ref), absum)
    assert float(np.max(np.abs(got - ref) / np.where(d > 0, d, 1.0))) <= 1e-5


@pytest.mark.parametrize("integer", [False, True])
def test_sw_stencil_exact(rt, torch_mod, integer):
    f = flep_mod()
    n = 1030
    a = gen.stencil_i32_input(n, seed=53) if integer else gen.stencil_f32_input(n, seed=53)
    body = f.BODY_STENCIL5_I32 if integer else f.BODY_STENCIL5_F32
    ind = t(a)
    o0, o1 = torch_mod.empty_like(ind), torch_mod.empty_like(ind)
    rt.launch_unwrapped(body, f.stencil_grid(n), f.stencil_args(o0, ind))
    k = rt.register_kernel(body, chunk=2, poll=1, sched_warp=True)
    h = rt.launch(k, f.stencil_grid(n), f.stencil_args(o1, ind))
    rt.sync(h, timeout_ns=10_000_000_000)
    torch_mod.cuda.synchronize()
    g = f.stencil_grid(n)
    assert np.all(rt.coverage_np(h, g[0] * g[1]) == 1)
    assert torch_mod.equal(o0.view(torch_mod.int32), o1.view(torch_mod.int32))
    if integer:
        assert np.array_equal(o1.cpu().numpy(), W.stencil5_i32(a))


@pytest.mark.parametrize("seed", range(4))
def test_sw_preempt_resume_schedules(rt, torch_mod, seed):
    f = flep_mod()
    n = 1 << 20
    x, y = gen.saxpy_i32_inputs(n, seed=54 + seed)
    nb = n // 256
    k = rt.register_kernel(f.BODY_SAXPY_I32, chunk=1 + seed % 2, poll=1, sched_warp=True)
    xd, yd = t(x), t(y)
    sched = gen.preempt_schedule(900 + seed, nb, rt.num_sms)
    h, npre, viol = run_manual_schedule(rt, k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, 3), nb, sched,
                                        rt.num_sms)
    assert viol == []
    assert np.all(rt.coverage_np(h, nb) == 1)
    assert np.array_equal(yd.cpu().numpy(), W.saxpy_i32(3, x, y))


def test_sw_rejected_for_tma_body(rt, torch_mod):
    f = flep_mod()
    ind = torch_mod.zeros((256, 256), device="cuda")
    outd = torch_mod.empty_like(ind)
    k = rt.register_kernel(f.BODY_STENCIL5_F32_TMA, chunk=1, poll=1, sched_warp=True)
    with pytest.raises(f.FlepError):
        rt.launch(k, f.stencil_grid(256), f.stencil_args(outd, ind))


def test_sw_random_schedules_2k_zero_violations(rt, torch_mod):
    """2 x 10^3 random manual preempt/resume schedules (config 1 generator) on the scheduling-warp
    worker: coverage == 1 after every schedule, I2 prefix and I3 on every 10th, exact results."""
    f = flep_mod()
    n, a = 1 << 20, 1664525
    nb = n // 256
    x, y = gen.saxpy_i32_inputs(n, seed=1)
    ref = W.saxpy_i32(a, x, y)
    xd, y0, yd = t(x), t(y), t(y)
    kern, bad, yielded = {}, [], 0
    for i in range(2000):
        s = gen.preempt_schedule(20_000 + i, nb, rt.num_sms)
        key = (s["C"], s["K"])
        if key not in kern:
            kern[key] = rt.register_kernel(f.BODY_SAXPY_I32, chunk=s["C"], poll=s["K"], sched_warp=True)
        yd.copy_(y0)
        h, npre, viol = run_manual_schedule(rt, kern[key], f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, a), nb,
                                            s, rt.num_sms, check_prefix=(i % 10 == 0))
        yielded += int(npre > 0)
        if not np.all(rt.coverage_np(h, nb) == 1):
            viol.append("I1: coverage != 1")
        if (i % 10 == 0 or viol) and not np.array_equal(yd.cpu().numpy(), ref):
            viol.append("result != oracle")
        if viol:
            bad.append((i, s, viol))
    assert bad == [], bad[:3]
    # the ring holds one chunk ahead, so large C*K schedules often finish before the request is
    # seen; enough of them still drain whole epochs (119 of 2000 on the B200)
    assert yielded > 50
