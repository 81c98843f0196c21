"""GPU parity of the wide CTA-pair GEMM body (FLEP_BODY_GEMM_BF16_2SM_W: a 256x512 output tile per
pair, two N = 256 tcgen05.mma.cta_group::2 per k-slice into one 512-column TMEM accumulator)
against the oracle (fp64 from the same bf16 inputs, MM P:286): unwrapped, static persistent and
FLEP pair workers agree bit for bit with each other and with the 256x256 pair body (same products
in the same k order per output element); manual preempt/resume schedules and in-tile
preemption (256 KiB spilled per CTA) stay bit-identical with every tile run once."""
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


@pytest.mark.parametrize("m,n,k,chunk", [(256, 512, 64, 1), (512, 1024, 128, 1), (768, 2048, 512, 2),
                                         (1024, 3584, 1024, 3)])
def test_gemm2w_all_forms_agree(rt, m, n, k, chunk):
    import torch
    f = flep_mod()
    a_bits, b_bits = gen.gemm_bf16_inputs(m, n, k, seed=260 + m)
    ref = W.gemm_bf16(a_bits, b_bits)
    A, B = _bf16(a_bits), _bf16(b_bits)
    grid = f.gemm2w_grid(m, n)
    Cu = torch.full((m, n), float("nan"), dtype=torch.bfloat16, device="cuda")
    rt.launch_unwrapped(f.BODY_GEMM_BF16_2SM_W, grid, f.gemm_args(Cu, A, B))
    torch.cuda.synchronize()
    got = _check(Cu, ref)
    assert np.isfinite(got).all()
    # the 256x256 pair body: the same per-element products and k order
    Cn = torch.full((m, n), float("nan"), dtype=torch.bfloat16, device="cuda")
    rt.launch_unwrapped(f.BODY_GEMM_BF16_2SM, f.gemm2_grid(m, n), f.gemm_args(Cn, A, B))
    torch.cuda.synchronize()
    assert torch.equal(Cn.view(torch.int16), Cu.view(torch.int16))
    Cs = torch.full((m, n), float("nan"), dtype=torch.bfloat16, device="cuda")
    rt.launch_static(f.BODY_GEMM_BF16_2SM_W, grid, f.gemm_args(Cs, A, B))
    torch.cuda.synchronize()
    assert torch.equal(Cs.view(torch.int16), Cu.view(torch.int16))
    Cw = torch.full((m, n), float("nan"), dtype=torch.bfloat16, device="cuda")
    kk = rt.register_kernel(f.BODY_GEMM_BF16_2SM_W, chunk=chunk, poll=1)
    h = rt.launch(kk, grid, f.gemm_args(Cw, A, B))
    rt.sync(h, timeout_ns=20_000_000_000)
    assert torch.equal(Cw.view(torch.int16), Cu.view(torch.int16))
    ntiles = grid[0] * grid[1]
    assert np.all(rt.coverage_np(h, ntiles) == 1)
    _, pairs = rt.workers_for(f.BODY_GEMM_BF16_2SM_W)
    assert rt.query(h).workers == min(pairs, -(-ntiles // chunk))


def test_gemm2w_identity_exact(rt):
    import torch
    f = flep_mod()
    m, n, k = 512, 1024, 1024
    a_bits, _ = gen.gemm_bf16_inputs(m, k, k, seed=270)
    eye = gen.round_to_bf16_bits(np.eye(n, k, dtype=np.float32))
    A, B = _bf16(a_bits), _bf16(eye)
    C = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    kk = rt.register_kernel(f.BODY_GEMM_BF16_2SM_W, chunk=1, poll=1)
    h = rt.launch(kk, f.gemm2w_grid(m, n), f.gemm_args(C, A, B))
    rt.sync(h, timeout_ns=20_000_000_000)
    assert np.array_equal(C.view(torch.int16).cpu().numpy().view(np.uint16), a_bits)   # C == A bit-exact


def test_gemm2w_rejects_bad_shapes(rt):
    import torch
    f = flep_mod()
    A = torch.zeros((256, 64), dtype=torch.bfloat16, device="cuda")
    B = torch.zeros((256, 64), dtype=torch.bfloat16, device="cuda")
    C = torch.zeros((256, 256), dtype=torch.bfloat16, device="cuda")
    kk = rt.register_kernel(f.BODY_GEMM_BF16_2SM_W, chunk=1, poll=1)
    with pytest.raises(f.FlepError):                  # N = 256 is not a multiple of 512
        rt.launch(kk, (1, 1, 1), f.gemm_args(C, A, B))


@pytest.mark.parametrize("seed", range(6))
def test_gemm2w_preempt_resume_schedules(rt, seed):
    """Random manual schedules (device triggers at random tiles, temporal and spatial widths):
    every tile exactly once, C bit-identical to the uninterrupted run, I3 on every epoch."""
    import torch
    f = flep_mod()
    m, n, k = 2048, 4096, 512
    a_bits, b_bits = gen.gemm_bf16_inputs(m, n, k, seed=271)
    A, B = _bf16(a_bits), _bf16(b_bits)
    grid = f.gemm2w_grid(m, n)
    ntiles = grid[0] * grid[1]
    C0 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    rt.launch_unwrapped(f.BODY_GEMM_BF16_2SM_W, grid, f.gemm_args(C0, A, B))
    torch.cuda.synchronize()
    sched = gen.preempt_schedule(2700 + seed, ntiles, rt.num_sms)
    kk = rt.register_kernel(f.BODY_GEMM_BF16_2SM_W, chunk=min(sched["C"], 4), poll=sched["K"])
    C1 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    h, npre, viol = run_manual_schedule(rt, kk, grid, f.gemm_args(C1, A, B), ntiles, sched, rt.num_sms,
                                        check_prefix=False)
    assert viol == []
    assert np.all(rt.coverage_np(h, ntiles) == 1)
    assert torch.equal(C1.view(torch.int16), C0.view(torch.int16))


def test_gemm2w_8192_sampled_vs_oracle(rt):
    """configs[3]'s largest GEMM (8192^3) through the wide pair workers: sampled rows against
    the oracle, and the whole C bit-identical to the 256x256 pair body."""
    import torch
    f = flep_mod()
    m = n = k = 8192
    g = torch.Generator(device="cuda")
    g.manual_seed(5)
    A = (torch.rand(m, k, device="cuda", generator=g) * 2 - 1).to(torch.bfloat16)
    B = (torch.rand(n, k, device="cuda", generator=g) * 2 - 1).to(torch.bfloat16)
    C = torch.empty(m, n, device="cuda", dtype=torch.bfloat16)
    kk = rt.register_kernel(f.BODY_GEMM_BF16_2SM_W, chunk=1, poll=1)
    h = rt.launch(kk, f.gemm2w_grid(m, n), f.gemm_args(C, A, B))
    rt.sync(h, timeout_ns=20_000_000_000)
    rows = [0, 1, 255, 256, 4097, 8191]
    a_bits = A[rows].view(torch.int16).cpu().numpy().view(np.uint16)
    b_bits = B.view(torch.int16).cpu().numpy().view(np.uint16)
    ref = W.gemm_bf16(a_bits, b_bits)
    got = C[rows].float().cpu().numpy().astype(np.float64)
    rms = float(np.sqrt(np.mean(ref ** 2)))
    assert np.all(np.abs(got - ref) <= TOL * (np.abs(ref) + rms))
    Cn = torch.empty(m, n, device="cuda", dtype=torch.bfloat16)
    rt.launch_unwrapped(f.BODY_GEMM_BF16_2SM, f.gemm2_grid(m, n), f.gemm_args(Cn, A, B))
    torch.cuda.synchronize()
    assert torch.equal(Cn.view(torch.int16), C.view(torch.int16))


@pytest.mark.parametrize("chunk", [1, 2])
def test_gemm2w_in_tile_random_schedules_bitexact(rt, chunk):
    """In-tile preemption on the wide pair: random temporal/spatial schedules stop pairs inside
    tiles (both 128x512 halves spilled, restored by the pair with the same index next epoch):
    every tile once, C bit-identical to the unwrapped grid, and some epochs really ended with
    tiles stopped mid-way."""
    import torch
    f = flep_mod()
    m, n, k = 2048, 4096, 4096                      # 64 tiles of 256x512, 64 k-steps each
    a_bits, b_bits = gen.gemm_bf16_inputs(m, n, k, seed=275 + chunk)
    A, B = _bf16(a_bits), _bf16(b_bits)
    grid = f.gemm2w_grid(m, n)
    ntiles = grid[0] * grid[1]
    C0 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    rt.launch_unwrapped(f.BODY_GEMM_BF16_2SM_W, grid, f.gemm_args(C0, A, B))
    torch.cuda.synchronize()
    _check(C0, W.gemm_bf16(a_bits, b_bits))
    kk = rt.register_kernel(f.BODY_GEMM_BF16_2SM_W, chunk=chunk, poll=1, in_tile=True)
    C1 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    stats, bad = {}, []
    for i in range(16):
        s = gen.preempt_schedule(2800 + 50 * chunk + i, ntiles, rt.num_sms)
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


def test_gemm2w_in_tile_latency_below_tile_time(rt):
    """A temporal request drains the in-tile wide pair GEMM in far less than one 256x512 tile's
    compute time (k = 8192: 128 k-steps per tile). 256 tiles (as the 256x256 test): with 128, the
    74 pairs finish their static first tiles within about a microsecond of each other and can
    fetch every remaining tile before the trigger's control word reaches them, so the
    tile-granular run may end DONE (a flake seen once in two suite runs)."""
    import torch
    f = flep_mod()
    m, n, k = 8192, 4096, 8192
    a_bits, b_bits = gen.gemm_bf16_inputs(m, n, k, seed=278)
    A, B = _bf16(a_bits), _bf16(b_bits)
    grid = f.gemm2w_grid(m, n)
    C0 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    rt.launch_unwrapped(f.BODY_GEMM_BF16_2SM_W, grid, f.gemm_args(C0, A, B))
    torch.cuda.synchronize()
    _, pairs = rt.workers_for(f.BODY_GEMM_BF16_2SM_W)
    C = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    out = {}
    for in_tile in (False, True):
        kk = rt.register_kernel(f.BODY_GEMM_BF16_2SM_W, chunk=1, poll=1, in_tile=in_tile)
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
            assert torch.equal(C.view(torch.int16), C0.view(torch.int16))
        out[in_tile] = float(np.median(lat))
    assert out[True] < 0.5 * out[False], out
