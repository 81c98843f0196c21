"""GPU parity: the CUDA path (through the C ABI) against the oracle, element by element, on the
same seeded inputs (SURVEY §8(c) "Parity criteria"). Bit-exact for integer work; fp32 within
1e-5 relative to the cancellation-safe denominator."""
import numpy as np
import pytest

from oracle import workloads as W
from synth import gen

from flep_gpu_util import flep_mod, run_manual_schedule, t

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


@pytest.mark.parametrize("n", [1, 255, 256, 1000, 4099, 1 << 16, (1 << 20) + 3])
@pytest.mark.parametrize("chunk,poll", [(1, 1), (8, 1), (16, 4)])
def test_saxpy_i32_wrapped_bitexact(rt, torch_mod, n, chunk, poll):
    f = flep_mod()
    x, y = gen.saxpy_i32_inputs(n, seed=1)
    a = 1664525
    ref = W.saxpy_i32(a, x, y)
    k = rt.register_kernel(f.BODY_SAXPY_I32, chunk=chunk, poll=poll)
    xd, yd = t(x), t(y)
    h = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, a))
    rt.sync(h)
    assert np.array_equal(yd.cpu().numpy(), ref)
    nb = f.saxpy_grid(n)[0]
    assert np.all(rt.coverage_np(h, nb) == 1)
    info = rt.query(h)
    assert info.state == f.STATE_DONE and info.blocks_done == nb
    # counter overshoot bounded by W*C (A5); uninterrupted: exactly ceil(N/C)*C + W*C
    assert info.counter == -(-nb // chunk) * chunk + info.workers * chunk


@pytest.mark.parametrize("n", [7, 256 * 37 + 5, 1 << 20])
def test_saxpy_f32_wrapped_and_unwrapped(rt, torch_mod, n):
    f = flep_mod()
    x, y = gen.saxpy_f32_inputs(n, seed=2)
    a = 0.75
    ref = W.saxpy_f32(a, x, y)
    k = rt.register_kernel(f.BODY_SAXPY_F32, chunk=4)
    xd, yd = t(x), t(y)
    h = rt.launch(k, f.saxpy_grid(n), f.saxpy_f32_args(yd, xd, a))
    rt.sync(h)
    got = yd.cpu().numpy()
    assert np.all(np.abs(got - ref) <= 1e-6 * (np.abs(a * x.astype(np.float64)) + np.abs(y)) + 1e-30)
    yd2 = t(y)
    rt.launch_unwrapped(f.BODY_SAXPY_F32, f.saxpy_grid(n), f.saxpy_f32_args(yd2, xd, a))
    torch_mod.cuda.synchronize()
    assert np.array_equal(yd2.cpu().numpy(), got)       # same body -> bit-identical


@pytest.mark.parametrize("rows,chunk", [(1, 1), (31, 2), (33, 1), (5000, 8), (1 << 16, 16)])
def test_spmv_wrapped_unwrapped(rt, torch_mod, rows, chunk):
    f = flep_mod()
    rowptr, col, val, x = gen.csr_inputs(rows, seed=3)
    ref, absum = W.spmv_csr(rowptr, col, val, x)
    k = rt.register_kernel(f.BODY_SPMV_CSR_F32, chunk=chunk)
    dr, dc, dv, dx = t(rowptr), t(col), t(val), t(x)
    yd = torch_mod.full((rows,), float("nan"), device="cuda")
    h = rt.launch(k, f.spmv_grid(rows), f.spmv_args(yd, dr, dc, dv, dx))
    rt.sync(h)
    got = yd.cpu().numpy()
    assert _rel_err(got, ref, absum) <= REL_FP32
    yd2 = torch_mod.full((rows,), float("nan"), device="cuda")
    rt.launch_unwrapped(f.BODY_SPMV_CSR_F32, f.spmv_grid(rows), f.spmv_args(yd2, dr, dc, dv, dx))
    torch_mod.cuda.synchronize()
    assert np.array_equal(yd2.cpu().numpy(), got)


@pytest.mark.parametrize("chunk", [1, 3, 8])
@pytest.mark.parametrize("variant", ["counter", "clc", "sched_warp"])
def test_spmv_empty_row_groups(rt, torch_mod, chunk, variant):
    """Runs of >= 256 consecutive empty rows (whole CSR-stream row groups without a nonzero) at
    the start, in the middle and at the end, at chunks that put several groups in one run (the
    ADVICE r1 race: an all-empty group skipped every barrier of the tile loop)."""
    f = flep_mod()
    rows = 6000
    runs = [(0, 300), (1000, 1800), (2304, 2816), (5600, 6000)]
    rowptr, col, val, x = gen.csr_inputs(rows, seed=13, empty_runs=runs)
    ref, absum = W.spmv_csr(rowptr, col, val, x)
    k = rt.register_kernel(f.BODY_SPMV_CSR_F32, chunk=chunk, poll=1, clc=variant == "clc",
                           sched_warp=variant == "sched_warp")
    dr, dc, dv, dx = t(rowptr), t(col), t(val), t(x)
    for _ in range(3):
        yd = torch_mod.full((rows,), float("nan"), device="cuda")
        h = rt.launch(k, f.spmv_grid(rows), f.spmv_args(yd, dr, dc, dv, dx))
        rt.sync(h)
        got = yd.cpu().numpy()
        assert _rel_err(got, ref, absum) <= REL_FP32
        for r0, r1 in runs:
            assert np.all(got[r0:r1] == 0.0)


@pytest.mark.parametrize("body", ["f32", "f32_tma"])
def test_stencil_16384_sampled_rows_vs_oracle(rt, torch_mod, body):
    """configs[2]'s victim size (16384^2, 2 GB in + out): every cell of sampled rows against the
    oracle, computed row by row on 3-row slabs (the middle row of a slab is an interior row with
    the same neighbours as in the full field; boundary rows are copied through)."""
    f = flep_mod()
    n = 16384
    a = gen.stencil_f32_input(n, seed=4)
    kb = f.BODY_STENCIL5_F32 if body == "f32" else f.BODY_STENCIL5_F32_TMA
    k = rt.register_kernel(kb, chunk=2, poll=1)
    ind = t(a)
    outd = torch_mod.empty_like(ind)
    h = rt.launch(k, f.stencil_grid(n), f.stencil_args(outd, ind))
    rt.sync(h)
    g = gen.rng(99)
    rows = sorted(set([1, 63, 64, 65, n - 2] + [int(r) for r in g.integers(1, n - 1, 40)]))
    for r in rows:
        ref, absum = W.stencil5_f32(a[r - 1:r + 2])
        got = outd[r].cpu().numpy()
        assert _rel_err(got, ref[1], absum[1]) <= REL_FP32, r
    for r in (0, n - 1):                                   # boundary rows: copied through
        assert np.array_equal(outd[r].cpu().numpy(), a[r])
    out2 = torch_mod.empty_like(ind)
    rt.launch_unwrapped(kb, f.stencil_grid(n), f.stencil_args(out2, ind))
    torch_mod.cuda.synchronize()
    assert torch_mod.equal(out2, outd)                      # wrapped == unwrapped, bit for bit


@pytest.mark.parametrize("n", [3, 64, 130, 257, 1000, 4096])
@pytest.mark.parametrize("integer", [False, True])
def test_stencil_wrapped_unwrapped(rt, torch_mod, n, integer):
    f = flep_mod()
    body = f.BODY_STENCIL5_I32 if integer else f.BODY_STENCIL5_F32
    a = gen.stencil_i32_input(n, seed=4) if integer else gen.stencil_f32_input(n, seed=4)
    k = rt.register_kernel(body, chunk=2)
    ind = t(a)
    outd = torch_mod.empty_like(ind)
    h = rt.launch(k, f.stencil_grid(n), f.stencil_args(outd, ind))
    rt.sync(h)
    got = outd.cpu().numpy()
    if integer:
        assert np.array_equal(got, W.stencil5_i32(a))
    else:
        ref, absum = W.stencil5_f32(a)
        assert _rel_err(got, ref, absum) <= REL_FP32
    out2 = torch_mod.empty_like(ind)
    rt.launch_unwrapped(body, f.stencil_grid(n), f.stencil_args(out2, ind))
    torch_mod.cuda.synchronize()
    assert np.array_equal(out2.cpu().numpy(), got)


def test_sliced_equals_wrapped(rt, torch_mod):
    f = flep_mod()
    n = 1 << 18
    x, y = gen.saxpy_i32_inputs(n, seed=5)
    xd = t(x)
    y1, y2 = t(y), t(y)
    rt.launch_sliced(f.BODY_SAXPY_I32, f.saxpy_grid(n), f.saxpy_i32_args(y1, xd, 3), 100)
    torch_mod.cuda.synchronize()
    assert np.array_equal(y1.cpu().numpy(), W.saxpy_i32(3, x, y))


def test_temporal_preempt_resume_bitexact(rt, torch_mod):
    """Config 1 shape: LP SAXPY-i32 2^20 preempted mid-run (device trigger), then resumed."""
    f = flep_mod()
    n = 1 << 20
    x, y = gen.saxpy_i32_inputs(n, seed=1)
    a = 1664525
    ref = W.saxpy_i32(a, x, y)
    nb = n // 256
    # W = 1184 workers and N = 4096 blocks: with C = K = 1 every worker polls between blocks
    k = rt.register_kernel(f.BODY_SAXPY_I32, chunk=1, poll=1)
    xd, yd = t(x), t(y)
    sched = {"cycles": [(nb // 3, rt.num_sms), (2 * nb // 3, rt.num_sms)]}
    h, npre, viol = run_manual_schedule(rt, k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, a), nb, sched,
                                        rt.num_sms)
    assert viol == []
    assert npre == 2
    assert np.all(rt.coverage_np(h, nb) == 1)
    assert np.array_equal(yd.cpu().numpy(), ref)


def test_spatial_yield_frees_exactly_requested_sms(rt, torch_mod):
    f = flep_mod()
    n = 4096
    a = gen.stencil_f32_input(n, seed=6)
    k = rt.register_kernel(f.BODY_STENCIL5_F32, chunk=1, poll=1)
    ind = t(a)
    outd = torch_mod.empty_like(ind)
    nb = (n // 64) ** 2
    for nsm in (8, 16, 32, 74):
        rt.arm_next_trigger(nb // 4, nsm)
        h = rt.launch(k, f.stencil_grid(n), f.stencil_args(outd, ind))
        rt.sync(h)
        ev = rt.events(h, 1)
        yielded = {e.smid for e in ev if e.reason == f.REASON_YIELD}
        kept = {e.smid for e in ev if e.reason == f.REASON_EXHAUSTED}
        assert yielded and max(yielded) < nsm          # only requested SMs yield (I3)
        assert min(kept) >= nsm                        # every worker elsewhere kept running
        assert all(e.reason != f.REASON_YIELD for e in ev if e.smid >= nsm)
        # every worker on a yielded SM left (they do not process blocks after the request)
        assert np.all(rt.coverage_np(h, nb) == 1)
        ref, absum = W.stencil5_f32(a)
        assert _rel_err(outd.cpu().numpy(), ref, absum) <= REL_FP32


def test_manual_api_errors(rt, torch_mod):
    f = flep_mod()
    n = 1 << 12
    x, y = gen.saxpy_i32_inputs(n, seed=7)
    k = rt.register_kernel(f.BODY_SAXPY_I32)
    xd, yd = t(x), t(y)
    h = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, 1))
    rt.sync(h)
    with pytest.raises(f.FlepError) as e:
        rt.preempt(h, rt.num_sms)
    assert e.value.status == f.ERR_STATE
    with pytest.raises(f.FlepError) as e:
        rt.resume(h)
    assert e.value.status == f.ERR_STATE
    with pytest.raises(f.FlepError) as e:
        rt.preempt(h, 0)
    assert e.value.status == f.ERR_INVALID
    with pytest.raises(f.FlepError) as e:
        rt.launch(k, (0, 1, 1), f.saxpy_i32_args(yd, xd, 1))
    assert e.value.status == f.ERR_INVALID
    with pytest.raises(f.FlepError) as e:
        rt.launch(999, (1, 1, 1), f.saxpy_i32_args(yd, xd, 1))
    assert e.value.status == f.ERR_INVALID
