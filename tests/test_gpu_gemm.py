"""GPU parity of the tcgen05 GEMM body (wrapped and unwrapped) against the oracle (fp64 from the
same bf16 inputs); preempt/resume at tile granularity (TMEM released before every exit)."""
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


@pytest.mark.parametrize("m,n,k,chunk", [(128, 256, 64, 1), (256, 512, 128, 1), (512, 1024, 512, 2),
                                         (1024, 1024, 1024, 3)])
def test_gemm_wrapped_unwrapped(rt, m, n, k, chunk):
    import torch
    f = flep_mod()
    a_bits, b_bits = gen.gemm_bf16_inputs(m, n, k, seed=60 + m)
    ref = W.gemm_bf16(a_bits, b_bits)
    A, B = _bf16(a_bits), _bf16(b_bits)
    C = torch.full((m, n), float("nan"), dtype=torch.bfloat16, device="cuda")
    kk = rt.register_kernel(f.BODY_GEMM_BF16, chunk=chunk, poll=1)
    h = rt.launch(kk, f.gemm_grid(m, n), f.gemm_args(C, A, B))
    rt.sync(h, timeout_ns=20_000_000_000)
    got = _check(C, ref)
    assert np.all(rt.coverage_np(h, (m // 128) * (n // 256)) == 1)
    C2 = torch.full((m, n), float("nan"), dtype=torch.bfloat16, device="cuda")
    rt.launch_unwrapped(f.BODY_GEMM_BF16, f.gemm_grid(m, n), f.gemm_args(C2, A, B))
    torch.cuda.synchronize()
    assert np.array_equal(C2.float().cpu().numpy(), got.astype(np.float32))   # same tile arithmetic


def test_gemm_identity_exact(rt):
    import torch
    f = flep_mod()
    m = n = k = 256
    a_bits, _ = gen.gemm_bf16_inputs(m, n, k, seed=70)
    eye = gen.round_to_bf16_bits(np.eye(n, k, dtype=np.float32))
    A, B = _bf16(a_bits), _bf16(eye)
    C = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    kk = rt.register_kernel(f.BODY_GEMM_BF16, chunk=1, poll=1)
    h = rt.launch(kk, f.gemm_grid(m, n), f.gemm_args(C, A, B))
    rt.sync(h, timeout_ns=20_000_000_000)
    assert np.array_equal(C.view(torch.int16).cpu().numpy().view(np.uint16), a_bits)   # C == A bit-exact


def test_gemm_preempt_resume_bitexact(rt):
    import torch
    f = flep_mod()
    m, n, k = 2048, 2048, 512
    a_bits, b_bits = gen.gemm_bf16_inputs(m, n, k, seed=71)
    A, B = _bf16(a_bits), _bf16(b_bits)
    C0 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    C1 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    ntiles = (m // 128) * (n // 256)
    kk = rt.register_kernel(f.BODY_GEMM_BF16, chunk=1, poll=1, ctas_per_sm=1)
    h0 = rt.launch(kk, f.gemm_grid(m, n), f.gemm_args(C0, A, B))
    rt.sync(h0, timeout_ns=20_000_000_000)
    for nsm in (rt.num_sms, 40):
        rt.arm_next_trigger(ntiles // 3, nsm)
        h = rt.launch(kk, f.gemm_grid(m, n), f.gemm_args(C1, A, B))
        rt.wait_epoch(h, timeout_ns=20_000_000_000)
        if rt.query(h).state == f.STATE_PREEMPTED:
            rt.resume(h)
        rt.sync(h, timeout_ns=20_000_000_000)
        assert np.all(rt.coverage_np(h, ntiles) == 1)
        assert torch.equal(C0.view(torch.int16), C1.view(torch.int16))
    ref = W.gemm_bf16(a_bits, b_bits)
    _check(C1, ref)


def test_gemm_full_size_sampled(rt):
    """BASELINE config 4's 8192^3 in the launch configuration the queue bench uses: sampled
    entries against the oracle computed one by one."""
    import torch
    f = flep_mod()
    m = n = k = 8192
    a_bits, b_bits = gen.gemm_bf16_inputs(m, n, k, seed=72)
    A, B = _bf16(a_bits), _bf16(b_bits)
    C = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    kk = rt.register_kernel(f.BODY_GEMM_BF16, chunk=1, poll=1)
    h = rt.launch(kk, f.gemm_grid(m, n), f.gemm_args(C, A, B))
    rt.sync(h, timeout_ns=60_000_000_000)
    Cn = C.float().cpu().numpy()
    g = gen.rng(73)
    rows, cols = g.integers(0, m, 256), g.integers(0, n, 256)
    ref = np.array([W.gemm_entry(a_bits, b_bits, r, c) for r, c in zip(rows, cols)])
    rms = float(np.sqrt(k / 9.0))       # rms of a sum of k products of U(-1,1) variables
    err = np.abs(Cn[rows, cols] - ref)
    assert np.all(err <= TOL * (np.abs(ref) + rms))


@pytest.mark.parametrize("chunk", [1, 2])
def test_gemm_in_tile_random_schedules_bitexact(rt, chunk):
    """In-tile preemption: random temporal/spatial preempt/resume schedules stop
    workers inside tiles (the accumulator is spilled and restored by the next epoch). Every
    schedule: coverage == 1, yields only on requested SMs, drained epochs cover a counter prefix,
    and C bit-identical to an uninterrupted run of the same binary."""
    import torch
    f = flep_mod()
    m, n, k = 1024, 2048, 4096                      # 64 tiles, 64 k-steps per tile
    ntiles = (m // 128) * (n // 256)
    a_bits, b_bits = gen.gemm_bf16_inputs(m, n, k, seed=80 + chunk)
    A, B = _bf16(a_bits), _bf16(b_bits)
    kk = rt.register_kernel(f.BODY_GEMM_BF16, chunk=chunk, poll=1, ctas_per_sm=1, in_tile=True,
                            async_poll=chunk == 2)
    C0 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    h0 = rt.launch(kk, f.gemm_grid(m, n), f.gemm_args(C0, A, B))
    rt.sync(h0, timeout_ns=20_000_000_000)
    _check(C0, W.gemm_bf16(a_bits, b_bits))
    C1 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    stats, bad = {}, []
    for i in range(40):
        s = gen.preempt_schedule(400 + i, ntiles, rt.num_sms)
        C1.fill_(float("nan"))
        h, npre, viol = run_manual_schedule(rt, kk, f.gemm_grid(m, n), f.gemm_args(C1, A, B), ntiles, s,
                                            rt.num_sms, stats=stats)
        if not np.all(rt.coverage_np(h, ntiles) == 1):
            viol.append("I1: coverage != 1")
        if not torch.equal(C0.view(torch.int16), C1.view(torch.int16)):
            viol.append("C differs from the uninterrupted run")
        if viol:
            bad.append((i, s, viol))
    assert not bad, bad[:3]
    assert stats.get("partial_epochs", 0) > 5       # tiles really were stopped mid-way


def test_gemm_in_tile_latency_below_tile_time(rt):
    """A temporal request drains an in-tile GEMM in far less than one tile's compute time."""
    import torch
    f = flep_mod()
    m = n = 4096
    k = 8192                                        # 128 k-steps per tile
    ntiles = (m // 128) * (n // 256)
    a_bits, b_bits = gen.gemm_bf16_inputs(m, n, k, seed=90)
    A, B = _bf16(a_bits), _bf16(b_bits)
    C = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
    out = {}
    for in_tile in (False, True):
        kk = rt.register_kernel(f.BODY_GEMM_BF16, chunk=1, poll=1, ctas_per_sm=1, in_tile=in_tile)
        lat = []
        for rep in range(3):
            rt.arm_next_trigger(rt.num_sms + 20, rt.num_sms)    # after the static first wave
            h = rt.launch(kk, f.gemm_grid(m, n), f.gemm_args(C, A, B))
            rt.wait_epoch(h, timeout_ns=20_000_000_000)
            assert rt.query(h).state == f.STATE_PREEMPTED
            ep = rt.epoch_info(h, 1)
            lat.append((ep.t_end - ep.t_trigger) / 1e3)
            rt.resume(h)
            rt.sync(h, timeout_ns=20_000_000_000)
        out[in_tile] = float(np.median(lat))
    assert out[True] < 0.5 * out[False], out
