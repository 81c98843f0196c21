"""GPU parity of the TMA-staged stencil body (FLEP_BODY_STENCIL5_F32_TMA): against the oracle
(fp32 tolerance of SURVEY §8(c)) and bit for bit against the register-path stencil body (same
per-cell arithmetic), for the unwrapped grid, the counter worker and the CLC worker, on tile-aligned
and ragged sizes; exactly-once under a preempt/resume schedule."""
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


@pytest.mark.parametrize("n", [4, 64, 1000, 1028, 4096])
@pytest.mark.parametrize("variant", ["unwrapped", "counter", "clc"])
def test_stencil_tma_matches_oracle_and_register_body(rt, torch_mod, n, variant):
    f = flep_mod()
    a = gen.stencil_f32_input(n, seed=41)
    ind = t(a)
    out_tma = torch_mod.full_like(ind, float("nan"))
    out_reg = torch_mod.full_like(ind, float("nan"))
    grid = f.stencil_grid(n)
    # register-path reference run (unwrapped grid of the plain body)
    rt.launch_unwrapped(f.BODY_STENCIL5_F32, grid, f.stencil_args(out_reg, ind))
    if variant == "unwrapped":
        rt.launch_unwrapped(f.BODY_STENCIL5_F32_TMA, grid, f.stencil_args(out_tma, ind))
    else:
        k = rt.register_kernel(f.BODY_STENCIL5_F32_TMA, chunk=2, poll=1, clc=variant == "clc")
        h = rt.launch(k, grid, f.stencil_args(out_tma, ind))
        rt.sync(h, timeout_ns=10_000_000_000)
        assert np.all(rt.coverage_np(h, grid[0] * grid[1]) == 1)
    torch_mod.cuda.synchronize()
    got = out_tma.cpu().numpy()
    ref, absum = W.stencil5_f32(a)
    assert _rel_err(got, ref, absum) <= REL_FP32
    assert np.array_equal(got.view(np.int32), out_reg.cpu().numpy().view(np.int32))


def test_stencil_tma_preempt_resume_exactly_once(rt, torch_mod):
    f = flep_mod()
    n = 4096
    a = gen.stencil_f32_input(n, seed=42)
    ind = t(a)
    outd = torch_mod.empty_like(ind)
    nb = (n // 64) ** 2
    k = rt.register_kernel(f.BODY_STENCIL5_F32_TMA, chunk=1, poll=1)
    sched = {"cycles": [(nb // 4, rt.num_sms), (nb // 2, 16), (3 * nb // 4, rt.num_sms)]}
    h, npre, viol = run_manual_schedule(rt, k, f.stencil_grid(n), f.stencil_args(outd, ind), nb, sched,
                                        rt.num_sms)
    assert viol == []
    assert np.all(rt.coverage_np(h, nb) == 1)
    ref, absum = W.stencil5_f32(a)
    assert _rel_err(outd.cpu().numpy(), ref, absum) <= REL_FP32


def test_stencil_tma_rejects_unaligned_rows(rt, torch_mod):
    f = flep_mod()
    ind = torch_mod.zeros((1030, 1030), device="cuda")
    outd = torch_mod.empty_like(ind)
    with pytest.raises(f.FlepError):
        rt.launch_unwrapped(f.BODY_STENCIL5_F32_TMA, f.stencil_grid(1030), f.stencil_args(outd, ind))
