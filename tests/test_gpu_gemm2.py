"""GPU parity of the CTA-pair GEMM body (FLEP_BODY_GEMM_BF16_2SM, tcgen05.mma.cta_group::2, R32)
against the oracle (fp64 from the same bf16 inputs): the unwrapped pair-per-tile grid, the static
persistent twin and the FLEP pair workers give bit-identical C; preempt/resume cycles (temporal
and spatial) stay bit-identical with every tile run once; a spatial request releases exactly the
pairs that have a named SM; with in-tile preemption (R21 + R32) the pair stops inside a tile,
spills both accumulator halves and the next epoch's pair continues it, bit-identically."""
import numpy as np
import pytest

from oracle import workloads as W
from synth import gen

from flep_gpu_util import flep_mod, run_manual_schedule

pytestmark = pytest.mark.gpu

TOL = 2e-2


def _bf16(bits):
    import torch
    return torch.from_numpy(bits.view(np.int16)).cuda().view(torch.bfloat16)


def _check(c_gpu, ref):
    got = c_gpu.float().cpu().numpy().astype(np.float64)
    rms = float(np.sqrt(np.mean(ref ** 2)))
    assert np.all(np.abs(got - ref) <= TOL * (np.abs(ref) + rms)), float(np.max(np.abs(got - ref)))
    assert np.linalg.norm(got - ref) <= TOL * np.linalg.norm(ref)
    return got


@pytest.fixture(scope="module")
def rt():
    f = flep_mod()
    r = f.Runtime(coverage=True)
    yield r
    r.close()


@pytest.mark.parametrize("m,n,k,chunk", [(256, 256, 64, 1), (256, 512, 128, 1), (512, 1024, 512, 2),
                                         (1024, 2048, 1024, 3)])
def test_gemm2_all_forms_agree(rt, m, n, k, chunk):
    import torch
    f = flep_mod()
    a_bits, b_bits = gen.gemm_bf16_inputs(m, n, k, seed=160 + m)
    ref = W.gemm_bf16(a_bits, b_bits)
    A, B = _bf16(a_bits), _bf16(b_bits)
    grid = f.gemm2_grid(m, n)
    Cu = torch.full((m, n), float("nan"), dtype=torch.bfloat16, device="cuda")
    rt.launch_unwrapped(f.BODY_GEMM_BF16_2SM, grid, f.gemm_args(Cu, A, B))
    torch.cuda.synchronize()
    got = _check(Cu, ref)
    Cs = torch.full((m, n), float("nan"), dtype=torch.bfloat16, device="cuda")
    rt.launch_static(f.BODY_GEMM_BF16_2SM, grid, f.gemm_args(Cs, A, B))
    torch.cuda.synchronize()
    assert torch.equal(Cs, Cu)
    Cw = torch.full((m, n), float("nan"), dtype=torch.bfloat16, device="cuda")
    kk = rt.register_kernel(f.BODY_GEMM_BF16_2SM, chunk=chunk, poll=1)
    h = rt.launch(kk, grid, f.gemm_args(Cw, A, B))
    rt.sync(h, timeout_ns=20_000_000_000)
    assert torch.equal(Cw, Cu)
    ntiles = grid[0] * grid[1]
    assert np.all(rt.coverage_np(h, ntiles) == 1)
    info = rt.query(h)
    _, pairs = rt.workers_for(f.BODY_GEMM_BF16_2SM)
    assert info.workers == min(pairs, -(-ntiles // chunk))
    assert np.isfinite(got).all()


def test_gemm2_identity_exact(rt):
    import torch
    f = flep_mod()
    m = n = k = 512
    a_bits, _ = gen.gemm_bf16_inputs(m, n, k, seed=170)
    eye = gen.round_to_bf16_bits(np.eye(n, k, dtype=np.float32))
    A, B = _bf16(a_bits), _bf16(eye)
    C = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    kk = rt.register_kernel(f.BODY_GEMM_BF16_2SM, chunk=1, poll=1)
    h = rt.launch(kk, f.gemm2_grid(m, n), f.gemm_args(C, A, B))
    rt.sync(h, timeout_ns=20_000_000_000)
    assert np.array_equal(C.view(torch.int16).cpu().numpy().view(np.uint16), a_bits)   # C == A bit-exact


@pytest.mark.parametrize("seed", range(8))
def test_gemm2_preempt_resume_schedules(rt, seed):
    """Random manual schedules (device triggers at random tiles, temporal and spatial widths):
    every tile exactly once, C bit-identical to the uninterrupted run, pairs yield only when a
    named SM is theirs (a pair's worker record names its lower-ranked SM, which decides, R32)."""
    import torch
    f = flep_mod()
    m, n, k = 2048, 2048, 512
    a_bits, b_bits = gen.gemm_bf16_inputs(m, n, k, seed=171)
    A, B = _bf16(a_bits), _bf16(b_bits)
    grid = f.gemm2_grid(m, n)
    ntiles = grid[0] * grid[1]
    C0 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    rt.launch_unwrapped(f.BODY_GEMM_BF16_2SM, grid, f.gemm_args(C0, A, B))
    torch.cuda.synchronize()
    sched = gen.preempt_schedule(1700 + seed, ntiles, rt.num_sms)
    kk = rt.register_kernel(f.BODY_GEMM_BF16_2SM, chunk=min(sched["C"], 4), poll=sched["K"])
    C1 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    h, npre, viol = run_manual_schedule(rt, kk, grid, f.gemm_args(C1, A, B), ntiles, sched, rt.num_sms,
                                        check_prefix=False)
    assert viol == []
    assert np.all(rt.coverage_np(h, ntiles) == 1)
    assert torch.equal(C1, C0)


def test_gemm2_8192_sampled_vs_oracle(rt):
    """configs[3]'s largest GEMM size (8192^3) through the pair workers: sampled output rows
    against the oracle (fp64 dot products of the same bf16 rows)."""
    import torch
    f = flep_mod()
    m = n = k = 8192
    g = torch.Generator(device="cuda")
    g.manual_seed(5)
    A = (torch.rand(m, k, device="cuda", generator=g) * 2 - 1).to(torch.bfloat16)
    B = (torch.rand(n, k, device="cuda", generator=g) * 2 - 1).to(torch.bfloat16)
    C = torch.empty(m, n, device="cuda", dtype=torch.bfloat16)
    kk = rt.register_kernel(f.BODY_GEMM_BF16_2SM, chunk=1, poll=1)
    h = rt.launch(kk, f.gemm2_grid(m, n), f.gemm_args(C, A, B))
    rt.sync(h, timeout_ns=20_000_000_000)
    rows = [0, 1, 255, 256, 4097, 8191]
    a_bits = A[rows].view(torch.int16).cpu().numpy().view(np.uint16)
    b_bits = B.view(torch.int16).cpu().numpy().view(np.uint16)
    ref = W.gemm_bf16(a_bits, b_bits)
    got = C[rows].float().cpu().numpy().astype(np.float64)
    rms = float(np.sqrt(np.mean(ref ** 2)))
    assert np.all(np.abs(got - ref) <= TOL * (np.abs(ref) + rms))


def test_gemm2_sliced_with_device_check_preempted():
    """Kernel slicing with the device check (R31) on the pair body: a higher-priority arrival
    makes the remaining slices skip; the resumed run is bit-identical to the unwrapped grid."""
    import torch
    f = flep_mod()
    rs = f.Runtime(policy=f.POLICY_SLICE_DEVICE, slice_blocks=16)
    try:
        m, n, k = 8192, 4096, 2048                 # ~0.1 ms: the arrival lands while it runs
        a_bits, b_bits = gen.gemm_bf16_inputs(m, n, k, seed=172)
        A, B = _bf16(a_bits), _bf16(b_bits)
        grid = f.gemm2_grid(m, n)
        C0 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
        rs.launch_unwrapped(f.BODY_GEMM_BF16_2SM, grid, f.gemm_args(C0, A, B))
        torch.cuda.synchronize()
        C1 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
        kl = rs.register_kernel(f.BODY_GEMM_BF16_2SM, chunk=1, poll=1, model=(0, 0, 0, 0, 2_000_000))
        kh = rs.register_kernel(f.BODY_SAXPY_I32, chunk=1, poll=1, model=(0, 0, 0, 0, 5_000))
        x, y = gen.saxpy_i32_inputs(1 << 16, seed=173)
        xd, yd = torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda()
        h1 = rs.launch(kl, grid, f.gemm_args(C1, A, B), priority=0)
        h2 = rs.launch(kh, f.saxpy_grid(1 << 16), f.saxpy_i32_args(yd, xd, 3), priority=1)
        rs.sync(h2, timeout_ns=20_000_000_000)
        rs.sync(h1, timeout_ns=20_000_000_000)
        torch.cuda.synchronize()
        assert torch.equal(C1, C0)
        assert np.array_equal(yd.cpu().numpy(), W.saxpy_i32(3, x, y))
        acts = [f.ACTION_NAMES[d[1]] for d in rs.decision_log()]
        assert acts[:3] == ["LAUNCH", "PREEMPT", "LAUNCH"]
    finally:
        rs.close()


@pytest.mark.parametrize("chunk", [1, 2])
def test_gemm2_in_tile_random_schedules_bitexact(rt, chunk):
    """In-tile preemption on the CTA pair: random temporal/spatial schedules stop pairs inside
    tiles (both 128-row halves spilled, restored by the pair with the same index next epoch).
    Every schedule: every tile once, C bit-identical to the unwrapped grid, and some epochs
    really ended with tiles stopped mid-way."""
    import torch
    f = flep_mod()
    m, n, k = 2048, 2048, 4096                      # 64 tiles of 256x256, 64 k-steps each
    a_bits, b_bits = gen.gemm_bf16_inputs(m, n, k, seed=175 + chunk)
    A, B = _bf16(a_bits), _bf16(b_bits)
    grid = f.gemm2_grid(m, n)
    ntiles = grid[0] * grid[1]
    C0 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    rt.launch_unwrapped(f.BODY_GEMM_BF16_2SM, grid, f.gemm_args(C0, A, B))
    torch.cuda.synchronize()
    _check(C0, W.gemm_bf16(a_bits, b_bits))
    kk = rt.register_kernel(f.BODY_GEMM_BF16_2SM, chunk=chunk, poll=1, in_tile=True)
    C1 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    stats, bad = {}, []
    for i in range(24):
        s = gen.preempt_schedule(1800 + 50 * chunk + i, ntiles, rt.num_sms)
        C1.fill_(float("nan"))
        h, npre, viol = run_manual_schedule(rt, kk, grid, f.gemm_args(C1, A, B), ntiles, s, rt.num_sms,
                                            check_prefix=False, stats=stats)
        if not np.all(rt.coverage_np(h, ntiles) == 1):
            viol.append("I1: coverage != 1")
        if not torch.equal(C0.view(torch.int16), C1.view(torch.int16)):
            viol.append("C differs from the uninterrupted run")
        if viol:
            bad.append((i, s, viol))
    assert not bad, bad[:3]
    assert stats.get("partial_epochs", 0) > 3       # tiles really were stopped mid-way


def test_gemm2_in_tile_latency_below_tile_time(rt):
    """A temporal request drains the in-tile pair GEMM in far less than one tile's compute time
    (k = 8192: 128 k-steps per 256x256 tile)."""
    import torch
    f = flep_mod()
    m = n = 4096
    k = 8192
    a_bits, b_bits = gen.gemm_bf16_inputs(m, n, k, seed=178)
    A, B = _bf16(a_bits), _bf16(b_bits)
    grid = f.gemm2_grid(m, n)
    C0 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    rt.launch_unwrapped(f.BODY_GEMM_BF16_2SM, grid, f.gemm_args(C0, A, B))
    torch.cuda.synchronize()
    _, pairs = rt.workers_for(f.BODY_GEMM_BF16_2SM)
    C = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    out = {}
    for in_tile in (False, True):
        kk = rt.register_kernel(f.BODY_GEMM_BF16_2SM, chunk=1, poll=1, in_tile=in_tile)
        lat = []
        for rep in range(3):
            rt.arm_next_trigger(pairs + 10, rt.num_sms)   # after the static first wave
            h = rt.launch(kk, grid, f.gemm_args(C, A, B))
            rt.wait_epoch(h, timeout_ns=20_000_000_000)
            assert rt.query(h).state == f.STATE_PREEMPTED
            ep = rt.epoch_info(h, 1)
            lat.append((ep.t_end - ep.t_trigger) / 1e3)
            rt.resume(h)
            rt.sync(h, timeout_ns=20_000_000_000)
            assert torch.equal(C, C0)
        out[in_tile] = float(np.median(lat))
    assert out[True] < 0.5 * out[False], out
