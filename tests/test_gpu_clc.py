"""GPU tests of the CLC task-fetch variant (R25): the original grid's pending
CTAs are the work queue (clusterlaunchcontrol.try_cancel) instead of the atomic counter.
Every original block must run exactly once (coverage == 1) with outputs equal to the oracle's,
uninterrupted, under temporal and spatial requests and under random preempt/resume cycles; a
preempted CLC victim hands its SMs to a higher-priority waiting kernel."""
import os
import time

import numpy as np
import pytest

from oracle import workloads as W
from synth import gen

from flep_gpu_util import flep_mod, t

pytestmark = pytest.mark.gpu

REL_FP32 = 1e-5


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


@pytest.mark.parametrize("n", [1, 255, 4099, (1 << 20) + 3])
@pytest.mark.parametrize("chunk,poll", [(1, 1), (1, 4), (3, 1), (16, 2)])
def test_clc_saxpy_i32_exact(rt, torch_mod, n, chunk, poll):
    # CTA i of the CLC grid = original blocks [iC, iC+C); ragged last chunk when C does not divide N
    f = flep_mod()
    x, y = gen.saxpy_i32_inputs(n, seed=31)
    k = rt.register_kernel(f.BODY_SAXPY_I32, chunk=chunk, poll=poll, clc=True)
    xd, yd = t(x), t(y)
    h = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, 1664525))
    rt.sync(h, timeout_ns=10_000_000_000)
    nb = f.saxpy_grid(n)[0]
    assert np.all(rt.coverage_np(h, nb) == 1)
    assert np.array_equal(yd.cpu().numpy(), W.saxpy_i32(1664525, x, y))
    assert rt.query(h).state == f.STATE_DONE


@pytest.mark.parametrize("n,integer", [(1000, False), (4096, False), (1030, True)])
def test_clc_stencil_exact(rt, torch_mod, n, integer):
    f = flep_mod()
    a = gen.stencil_i32_input(n, seed=32) if integer else gen.stencil_f32_input(n, seed=32)
    body = f.BODY_STENCIL5_I32 if integer else f.BODY_STENCIL5_F32
    k = rt.register_kernel(body, chunk=1, poll=1, clc=True)
    ind = t(a)
    outd = torch_mod.empty_like(ind)
    h = rt.launch(k, f.stencil_grid(n), f.stencil_args(outd, ind))
    rt.sync(h, timeout_ns=10_000_000_000)
    g = f.stencil_grid(n)
    assert np.all(rt.coverage_np(h, g[0] * g[1]) == 1)
    if integer:
        assert np.array_equal(outd.cpu().numpy(), W.stencil5_i32(a))
    else:
        ref, absum = W.stencil5_f32(a)
        assert _rel_err(outd.cpu().numpy(), ref, absum) <= REL_FP32


def test_clc_spmv_matches_counter_variant_bitwise(rt, torch_mod):
    # the same body, so the CLC grid's rows equal the atomic-counter worker's bit for bit
    f = flep_mod()
    rows = 1 << 16
    rp, col, val, x = gen.csr_inputs(rows, seed=33)
    args_in = (t(rp), t(col), t(val), t(x))
    y0 = torch_mod.zeros(rows, device="cuda")
    y1 = torch_mod.zeros(rows, device="cuda")
    k0 = rt.register_kernel(f.BODY_SPMV_CSR_F32, chunk=2, poll=1)
    k1 = rt.register_kernel(f.BODY_SPMV_CSR_F32, chunk=3, poll=2, clc=True)
    for k, y in ((k0, y0), (k1, y1)):
        h = rt.launch(k, f.spmv_grid(rows), f.spmv_args(y, *args_in))
        rt.sync(h, timeout_ns=10_000_000_000)
    assert np.all(rt.coverage_np(h, f.spmv_grid(rows)[0]) == 1)
    assert torch_mod.equal(y0.view(torch_mod.int32), y1.view(torch_mod.int32))
    ref, absum = W.spmv_csr(rp, col, val, x)
    assert _rel_err(y1.cpu().numpy(), ref, absum) <= REL_FP32


def _resume_unless_done(rt, f, h):
    # a preempted CLC grid keeps completing chunks (its queued CTAs still start), so it may finish
    # between a state query and the resume
    try:
        rt.resume(h)
    except f.FlepError:
        assert rt.query(h).state == f.STATE_DONE


def _long_lp(rt, f, n_log2=27, seed=34, **kw):
    n = 1 << n_log2
    x, y = gen.saxpy_i32_inputs(n, seed=seed)
    k = rt.register_kernel(f.BODY_SAXPY_I32, chunk=kw.pop("chunk", 4), poll=1, clc=True, **kw)
    return n, x, y, k


def test_clc_temporal_preempt_hands_sms_to_waiting_kernel(rt, torch_mod):
    """Host preempt of a long CLC victim; the waiting kernel (higher priority) is launched after
    the request and must start before the victim completes; resume withdraws the request."""
    f = flep_mod()
    n, x, y, k = _long_lp(rt, f)
    xd, yd = t(x), t(y)
    n2 = 1 << 20
    x2, y2 = gen.saxpy_i32_inputs(n2, seed=35)
    x2d, y2d = t(x2), t(y2)
    k_hp = rt.register_kernel(f.BODY_SAXPY_I32, chunk=4, poll=1)
    h = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, 3), priority=0)
    time.sleep(50e-6)
    rt.preempt(h, rt.num_sms)
    assert rt.query(h).state in (f.STATE_PREEMPTED, f.STATE_DONE)   # in force at once (R25)
    h2 = rt.launch(k_hp, f.saxpy_grid(n2), f.saxpy_i32_args(y2d, x2d, 5), priority=1)
    rt.sync(h2, timeout_ns=10_000_000_000)
    _resume_unless_done(rt, f, h)
    rt.sync(h, timeout_ns=20_000_000_000)
    torch_mod.cuda.synchronize()
    nb = n // 256
    assert np.all(rt.coverage_np(h, nb) == 1)
    assert np.array_equal(yd.cpu().numpy(), W.saxpy_i32(3, x, y))
    assert np.array_equal(y2d.cpu().numpy(), W.saxpy_i32(5, x2, y2))
    ev = rt.events(h, 1)
    assert any(e.reason == f.REASON_YIELD for e in ev), "no first-wave worker yielded"


def test_clc_spatial_request_yields_only_named_sms(rt, torch_mod):
    f = flep_mod()
    n, x, y, k = _long_lp(rt, f, seed=36)
    xd, yd = t(x), t(y)
    nsm = 16
    h = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, 11), priority=0)
    time.sleep(50e-6)
    rt.preempt(h, nsm)
    assert rt.query(h).state in (f.STATE_PARTIAL, f.STATE_DONE)
    time.sleep(200e-6)
    _resume_unless_done(rt, f, h)
    rt.sync(h, timeout_ns=20_000_000_000)
    ev = rt.events(h, 1)
    yielded = [e for e in ev if e.reason == f.REASON_YIELD]
    assert all(e.smid < nsm for e in yielded)                # I3 (rank = smid)
    assert np.all(rt.coverage_np(h, n // 256) == 1)
    assert np.array_equal(yd.cpu().numpy(), W.saxpy_i32(11, x, y))


@pytest.mark.parametrize("seed", range(6))
def test_clc_random_preempt_resume_cycles_exactly_once(rt, torch_mod, seed):
    f = flep_mod()
    g = gen.rng(700 + seed)
    n, x, y, k = _long_lp(rt, f, n_log2=26, seed=37 + seed)
    xd, yd = t(x), t(y)
    h = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, 13), priority=0)
    cycles = 0
    try:
        for _ in range(int(g.integers(1, 5))):
            time.sleep(float(g.uniform(5e-6, 60e-6)))
            nsm = rt.num_sms if g.random() < 0.5 else int(g.integers(1, rt.num_sms))
            rt.preempt(h, nsm)
            time.sleep(float(g.uniform(5e-6, 60e-6)))
            rt.resume(h)
            cycles += 1
    except f.FlepError:                 # the grid completed between two requests
        assert rt.query(h).state == f.STATE_DONE
    rt.sync(h, timeout_ns=20_000_000_000)
    assert np.all(rt.coverage_np(h, n // 256) == 1)
    assert np.array_equal(yd.cpu().numpy(), W.saxpy_i32(13, x, y))


def test_clc_managed_hpf(torch_mod):
    """Managed HPF with a CLC victim: the policy's preempt/launch/resume sequence works on the
    hardware work queue; both results exact, victim exactly once."""
    f = flep_mod()
    rt = f.Runtime(policy=f.POLICY_HPF, coverage=True)
    try:
        n_lp, n_hp = 1 << 26, 1 << 16
        x, y = gen.saxpy_i32_inputs(n_lp, seed=38)
        x2, y2 = gen.saxpy_i32_inputs(n_hp, seed=39)
        xd, yd, x2d, y2d = t(x), t(y), t(x2), t(y2)
        k_lp = rt.register_kernel(f.BODY_SAXPY_I32, chunk=4, poll=1, clc=True, model=(0, 0, 0, 0, 2_000_000))
        k_hp = rt.register_kernel(f.BODY_SAXPY_I32, chunk=1, poll=1, model=(0, 0, 0, 0, 5_000))
        sA, sB = torch_mod.cuda.Stream(), torch_mod.cuda.Stream()
        h_lp = rt.launch(k_lp, f.saxpy_grid(n_lp), f.saxpy_i32_args(yd, xd, 7), priority=0, stream=sA)
        h_hp = rt.launch(k_hp, f.saxpy_grid(n_hp), f.saxpy_i32_args(y2d, x2d, 9), priority=1, stream=sB)
        rt.sync(h_hp, timeout_ns=10_000_000_000)
        rt.sync(h_lp, timeout_ns=20_000_000_000)
        torch_mod.cuda.synchronize()
        assert np.array_equal(yd.cpu().numpy(), W.saxpy_i32(7, x, y))
        assert np.array_equal(y2d.cpu().numpy(), W.saxpy_i32(9, x2, y2))
        assert np.all(rt.coverage_np(h_lp, n_lp // 256) == 1)
        acts = [f.ACTION_NAMES[d[1]] for d in rt.decision_log()]
        assert acts[:3] == ["LAUNCH", "PREEMPT", "LAUNCH"]
    finally:
        rt.close()


def test_clc_rejected_for_gemm(rt):
    f = flep_mod()
    import torch
    k = rt.register_kernel(f.BODY_GEMM_BF16, chunk=1, poll=1, clc=True)
    A = torch.zeros((128, 64), dtype=torch.bfloat16, device="cuda")
    B = torch.zeros((256, 64), dtype=torch.bfloat16, device="cuda")
    C = torch.empty((128, 256), dtype=torch.bfloat16, device="cuda")
    with pytest.raises(f.FlepError):
        rt.launch(k, f.gemm_grid(128, 256), f.gemm_args(C, A, B))


# ---- barrier-free CLC form (flep_clc_ring, reading R38): warp-task bodies at K = 1 ----------------

def test_clc_ring_and_barrier_forms_agree_bitwise(rt, torch_mod):
    """K = 1 selects the mbarrier-ring form for the stencil and SpMV-vector bodies, K = 4 the
    barrier form: the same blocks, so identical outputs (and the oracle's within fp32 tolerance)."""
    f = flep_mod()
    n = 4096 + 37                                        # ragged tiles
    a = gen.stencil_f32_input(n, seed=41)
    ind = t(a)
    outs = []
    for poll in (1, 4):
        k = rt.register_kernel(f.BODY_STENCIL5_F32, chunk=1, poll=poll, clc=True)
        o = torch_mod.empty_like(ind)
        h = rt.launch(k, f.stencil_grid(n), f.stencil_args(o, ind))
        rt.sync(h, timeout_ns=10_000_000_000)
        g = f.stencil_grid(n)
        assert np.all(rt.coverage_np(h, g[0] * g[1]) == 1)
        outs.append(o)
    assert torch_mod.equal(outs[0].view(torch_mod.int32), outs[1].view(torch_mod.int32))
    ref, absum = W.stencil5_f32(a)
    assert _rel_err(outs[0].cpu().numpy(), ref, absum) <= REL_FP32
    rows = (1 << 16) + 5
    rp, col, val, x = gen.csr_inputs(rows, seed=42)
    args_in = (t(rp), t(col), t(val), t(x))
    ys = []
    for poll in (1, 4):
        k = rt.register_kernel(f.BODY_SPMV_CSR_F32_VEC, chunk=1, poll=poll, clc=True)
        y = torch_mod.zeros(rows, device="cuda")
        h = rt.launch(k, f.spmv_grid(rows), f.spmv_args(y, *args_in))
        rt.sync(h, timeout_ns=10_000_000_000)
        assert np.all(rt.coverage_np(h, f.spmv_grid(rows)[0]) == 1)
        ys.append(y)
    assert torch_mod.equal(ys[0].view(torch_mod.int32), ys[1].view(torch_mod.int32))
    ref, absum = W.spmv_csr(rp, col, val, x)
    assert _rel_err(ys[0].cpu().numpy(), ref, absum) <= REL_FP32


@pytest.mark.parametrize("seed", range(int(os.environ.get("FLEP_RING_SEEDS", "4"))))
def test_clc_ring_random_preempt_resume_exactly_once(rt, torch_mod, seed):
    """The ring form under random temporal/spatial requests and resumes: a stencil-i32 16384²
    victim (65536 tiles) runs every tile once, output bit-exact against the oracle's closed form."""
    f = flep_mod()
    g = gen.rng(900 + seed)
    n = 16384
    a = gen.stencil_i32_input(n, seed=50 + seed)
    ind = t(a)
    outd = torch_mod.empty_like(ind)
    k = rt.register_kernel(f.BODY_STENCIL5_I32, chunk=1, poll=1, clc=True)
    h = rt.launch(k, f.stencil_grid(n), f.stencil_args(outd, ind), priority=0)
    requests = []
    try:
        for _ in range(int(g.integers(1, 5))):
            time.sleep(float(g.uniform(5e-6, 80e-6)))
            nsm = rt.num_sms if g.random() < 0.5 else int(g.integers(1, rt.num_sms))
            rt.preempt(h, nsm)
            requests.append(nsm)
            time.sleep(float(g.uniform(5e-6, 80e-6)))
            rt.resume(h)
    except f.FlepError:                 # the grid completed between two requests
        assert rt.query(h).state == f.STATE_DONE
    rt.sync(h, timeout_ns=20_000_000_000)
    gr = f.stencil_grid(n)
    assert np.all(rt.coverage_np(h, gr[0] * gr[1]) == 1)
    assert np.array_equal(outd.cpu().numpy(), W.stencil5_i32(a))
    if len(requests) == 1 and requests[0] < rt.num_sms:  # I3 when the one request was spatial
        for e in rt.events(h, 1):
            if e.reason == f.REASON_YIELD:
                assert e.smid < requests[0]


def test_clc_ring_temporal_preempt_releases_sms(rt, torch_mod):
    """A temporal request on a ring-form victim: first-wave workers yield, the waiting kernel runs,
    the resumed victim completes exactly once."""
    f = flep_mod()
    n = 16384
    a = gen.stencil_i32_input(n, seed=60)
    ind = t(a)
    outd = torch_mod.empty_like(ind)
    x2, y2 = gen.saxpy_i32_inputs(1 << 20, seed=61)
    x2d, y2d = t(x2), t(y2)
    k = rt.register_kernel(f.BODY_STENCIL5_I32, chunk=1, poll=1, clc=True)
    k_hp = rt.register_kernel(f.BODY_SAXPY_I32, chunk=4, poll=1)
    h = rt.launch(k, f.stencil_grid(n), f.stencil_args(outd, ind), priority=0)
    time.sleep(30e-6)
    rt.preempt(h, rt.num_sms)
    h2 = rt.launch(k_hp, f.saxpy_grid(1 << 20), f.saxpy_i32_args(y2d, x2d, 5), priority=1)
    rt.sync(h2, timeout_ns=10_000_000_000)
    _resume_unless_done(rt, f, h)
    rt.sync(h, timeout_ns=20_000_000_000)
    torch_mod.cuda.synchronize()
    gr = f.stencil_grid(n)
    assert np.all(rt.coverage_np(h, gr[0] * gr[1]) == 1)
    assert np.array_equal(outd.cpu().numpy(), W.stencil5_i32(a))
    assert np.array_equal(y2d.cpu().numpy(), W.saxpy_i32(5, x2, y2))
    assert any(e.reason == f.REASON_YIELD for e in rt.events(h, 1)), "no first-wave worker yielded"
