"""GPU tests of a user-defined body (include/flep_body.cuh, flep_register_body;
tests/user_body/body_affine_rev.cu): the FLEP worker, the original grid and the static twin that
FLEP_DEFINE_BODY instantiates in the user's own library agree exactly with a NumPy definition of
the body; random manual preempt/resume schedules (temporal and spatial yields, C and K random) run
every original block exactly once with an exact result and I3 on every epoch; under the managed
HPF policy a user-body kernel is preempted by a built-in higher-priority kernel and both results
are exact."""
import ctypes as C
import os

import numpy as np
import pytest

from oracle import workloads as W
from synth import gen

from flep_gpu_util import flep_mod, run_manual_schedule

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "tests", "user_body", "body_affine_rev.cu")
OUT = os.path.join(ROOT, "tests", "user_body", "build", "libaffine_rev.so")
PER = 512


class AffineRevArgs(C.Structure):
    _fields_ = [("y", C.c_void_p), ("x", C.c_void_p), ("a", C.c_int32), ("c", C.c_int32), ("n", C.c_uint32)]


def affine_rev_ref(x, a, c):
    """y[i] = a * x[mirror(i)] + c * block(i) (mod 2^32), mirror within the 512-element block,
    x beyond n read as 0 (the body's definition, int64 arithmetic wrapped to int32)."""
    n = len(x)
    nb = -(-n // PER)
    xp = np.zeros(nb * PER, dtype=np.int64)
    xp[:n] = x
    mir = xp.reshape(nb, PER)[:, ::-1].reshape(-1)[:n]
    blk = np.arange(n, dtype=np.int64) // PER
    return ((a * mir + c * blk) & 0xFFFFFFFF).astype(np.uint32).view(np.int32)


@pytest.fixture(scope="module")
def env():
    from paper_conf_asplos_wulzj17_b200 import build
    f = flep_mod()
    path = build.build_user_body(SRC, OUT)
    rt = f.Runtime(coverage=True)
    body = rt.register_body(path, "affine_rev")
    yield f, rt, body
    rt.close()


def _case(n, seed):
    import torch
    x, _ = gen.saxpy_i32_inputs(n, seed)
    xd = torch.from_numpy(x).cuda()
    yd = torch.zeros(n, dtype=torch.int32, device="cuda")
    args = AffineRevArgs(yd.data_ptr(), xd.data_ptr(), 1664525, 1013904223, n)
    return x, xd, yd, args


def test_register_returns_a_user_body_id(env):
    f, rt, body = env
    assert f.BODY_USER_FIRST <= body < f.BODY_USER_FIRST + 16


@pytest.mark.parametrize("n,chunk", [(512, 1), (100_000, 1), (1 << 20, 2), ((1 << 20) + 333, 3)])
def test_all_forms_match_the_definition(env, n, chunk):
    import torch
    f, rt, body = env
    x, xd, yd, args = _case(n, seed=900 + chunk)
    ref = affine_rev_ref(x, 1664525, 1013904223)
    grid = (-(-n // PER), 1, 1)
    rt.launch_unwrapped(body, grid, args)
    torch.cuda.synchronize()
    assert np.array_equal(yd.cpu().numpy(), ref)
    yd.zero_()
    rt.launch_static(body, grid, args, chunk=chunk)
    torch.cuda.synchronize()
    assert np.array_equal(yd.cpu().numpy(), ref)
    yd.zero_()
    k = rt.register_kernel(body, chunk=chunk, poll=1)
    h = rt.launch(k, grid, args)
    rt.sync(h, timeout_ns=20_000_000_000)
    assert np.array_equal(yd.cpu().numpy(), ref)
    assert np.all(rt.coverage_np(h, grid[0]) == 1)


@pytest.mark.parametrize("seed", range(40))
def test_random_preempt_resume_schedules_exact(env, seed):
    import torch
    f, rt, body = env
    n = (1 << 21) + 77
    x, xd, yd, args = _case(n, seed=950)
    ref = affine_rev_ref(x, 1664525, 1013904223)
    grid = (-(-n // PER), 1, 1)
    sched = gen.preempt_schedule(3100 + seed, grid[0], rt.num_sms)
    k = rt.register_kernel(body, chunk=sched["C"], poll=sched["K"])
    h, npre, viol = run_manual_schedule(rt, k, grid, args, grid[0], sched, rt.num_sms)
    assert viol == []
    assert np.all(rt.coverage_np(h, grid[0]) == 1)
    torch.cuda.synchronize()
    assert np.array_equal(yd.cpu().numpy(), ref)


def test_managed_hpf_preempts_a_user_body_kernel():
    import torch
    f = flep_mod()
    from paper_conf_asplos_wulzj17_b200 import build
    rs = f.Runtime(policy=f.POLICY_HPF, coverage=True)
    try:
        body = rs.register_body(build.build_user_body(SRC, OUT), "affine_rev")
        n = 1 << 26                                   # ~0.1 ms: the HP arrival lands while it runs
        x, xd, yd, args = _case(n, seed=960)
        grid = (-(-n // PER), 1, 1)
        kl = rs.register_kernel(body, chunk=1, poll=1, model=(0, 0, 0, 0, 5_000_000))
        kh = rs.register_kernel(f.BODY_SAXPY_I32, chunk=1, poll=1, model=(0, 0, 0, 0, 5_000))
        x2, y2 = gen.saxpy_i32_inputs(1 << 16, seed=961)
        x2d, y2d = torch.from_numpy(x2).cuda(), torch.from_numpy(y2).cuda()
        h1 = rs.launch(kl, grid, args, priority=0)
        h2 = rs.launch(kh, f.saxpy_grid(1 << 16), f.saxpy_i32_args(y2d, x2d, 7), priority=1)
        rs.sync(h2, timeout_ns=20_000_000_000)
        rs.sync(h1, timeout_ns=20_000_000_000)
        torch.cuda.synchronize()
        assert np.array_equal(yd.cpu().numpy(), affine_rev_ref(x, 1664525, 1013904223))
        assert np.array_equal(y2d.cpu().numpy(), W.saxpy_i32(7, x2, y2))
        acts = [f.ACTION_NAMES[d[1]] for d in rs.decision_log()]
        assert acts[:3] == ["LAUNCH", "PREEMPT", "LAUNCH"]
        assert np.all(rs.coverage_np(h1, grid[0]) == 1)
    finally:
        rs.close()


def test_args_size_mismatch_is_rejected(env):
    f, rt, body = env
    k = rt.register_kernel(body, chunk=1, poll=1)
    with pytest.raises(f.FlepError):                 # a 24-byte SAXPY struct for a 32-byte body
        rt.launch(k, (4, 1, 1), f.SaxpyI32Args(0, 0, 1, 0))


@pytest.mark.parametrize("chunk", [1, 4])
def test_clc_worker_of_a_user_body(env, chunk):
    """The CLC fetch (hardware work queue, R25) instantiated for the user body: exact result,
    every block once, also across host-issued preempt/resume cycles."""
    import time
    import torch
    f, rt, body = env
    n = 1 << 24
    x, xd, yd, args = _case(n, seed=970 + chunk)
    grid = (-(-n // PER), 1, 1)
    k = rt.register_kernel(body, chunk=chunk, poll=1, clc=True)
    h = rt.launch(k, grid, args)
    g = gen.rng(971 + chunk)
    try:
        for _ in range(3):
            time.sleep(float(g.uniform(5e-6, 40e-6)))
            rt.preempt(h, rt.num_sms if g.random() < 0.5 else int(g.integers(1, rt.num_sms)))
            time.sleep(float(g.uniform(5e-6, 40e-6)))
            rt.resume(h)
    except f.FlepError:                              # the grid completed between two requests
        assert rt.query(h).state == f.STATE_DONE
    rt.sync(h, timeout_ns=20_000_000_000)
    torch.cuda.synchronize()
    assert np.all(rt.coverage_np(h, grid[0]) == 1)
    assert np.array_equal(yd.cpu().numpy(), affine_rev_ref(x, 1664525, 1013904223))


def test_device_checked_slicing_of_a_user_body():
    """FLEP_POLICY_SLICE_DEVICE (R31) with the user body's slice kernel: a higher-priority arrival
    makes the remaining slices skip, the resumed slices finish the grid, results exact."""
    import torch
    from paper_conf_asplos_wulzj17_b200 import build
    f = flep_mod()
    rs = f.Runtime(policy=f.POLICY_SLICE_DEVICE, slice_blocks=2048)
    try:
        body = rs.register_body(build.build_user_body(SRC, OUT), "affine_rev")
        n = 1 << 26
        x, xd, yd, args = _case(n, seed=980)
        grid = (-(-n // PER), 1, 1)
        kl = rs.register_kernel(body, chunk=1, poll=1, model=(0, 0, 0, 0, 5_000_000))
        kh = rs.register_kernel(f.BODY_SAXPY_I32, chunk=1, poll=1, model=(0, 0, 0, 0, 5_000))
        x2, y2 = gen.saxpy_i32_inputs(1 << 16, seed=981)
        x2d, y2d = torch.from_numpy(x2).cuda(), torch.from_numpy(y2).cuda()
        h1 = rs.launch(kl, grid, args, priority=0)
        h2 = rs.launch(kh, f.saxpy_grid(1 << 16), f.saxpy_i32_args(y2d, x2d, 5), priority=1)
        rs.sync(h2, timeout_ns=20_000_000_000)
        rs.sync(h1, timeout_ns=20_000_000_000)
        torch.cuda.synchronize()
        assert np.array_equal(yd.cpu().numpy(), affine_rev_ref(x, 1664525, 1013904223))
        assert np.array_equal(y2d.cpu().numpy(), W.saxpy_i32(5, x2, y2))
        acts = [f.ACTION_NAMES[d[1]] for d in rs.decision_log()]
        assert acts[:3] == ["LAUNCH", "PREEMPT", "LAUNCH"]
    finally:
        rs.close()
