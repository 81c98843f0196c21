"""GPU tests of the runtime: the managed policies on real kernels (with replay parity of the
measured event log against the oracle DES), the 10^4 random preempt/resume schedules of config 1
(0 coverage violations, bit-exact results), the host-mapped flag transport, cancellation."""
import numpy as np
import pytest

from oracle import des
from oracle import workloads as W
from synth import gen

from flep_gpu_util import flep_mod, run_manual_schedule, t

pytestmark = pytest.mark.gpu

ACT = {"LAUNCH": 0, "RESUME": 1, "PREEMPT": 2}


def _replay_from_runtime(rt, kind):
    """Rebuild the oracle's event list from the runtime's own log and replay it."""
    evs = []
    for (t_ns, typ, lid, prio, t_e, ovh) in rt.event_log():
        if typ == 0:
            evs.append((t_ns, "ARRIVE", des.KernelSpec(lid, t_ns, prio, t_e, ovh)))
        else:
            evs.append((t_ns, "FINISH", lid))
    return [(t, ACT[a], i, n) for (t, a, i, n) in des.replay(kind, evs)]


def test_managed_hpf_preempts_and_replays_exactly():
    f = flep_mod()
    import torch
    rt = f.Runtime(policy=f.POLICY_HPF, coverage=True)
    try:
        n_lp, n_hp = 1 << 26, 1 << 16
        x, y = gen.saxpy_i32_inputs(n_lp, seed=21)
        x2, y2 = gen.saxpy_i32_inputs(n_hp, seed=22)
        xd, yd, x2d, y2d = t(x), t(y), t(x2), t(y2)
        k_lp = rt.register_kernel(f.BODY_SAXPY_I32, chunk=4, poll=1, model=(0, 0, 0, 0, 2_000_000))
        k_hp = rt.register_kernel(f.BODY_SAXPY_I32, chunk=1, poll=1, model=(0, 0, 0, 0, 5_000))
        sA, sB = torch.cuda.Stream(), torch.cuda.Stream()
        h_lp = rt.launch(k_lp, f.saxpy_grid(n_lp), f.saxpy_i32_args(yd, xd, 7), priority=0, stream=sA)
        h_hp = rt.launch(k_hp, f.saxpy_grid(n_hp), f.saxpy_i32_args(y2d, x2d, 9), priority=1, stream=sB)
        rt.sync(h_hp, timeout_ns=10_000_000_000)
        rt.sync(h_lp, timeout_ns=10_000_000_000)
        torch.cuda.synchronize()
        assert np.array_equal(yd.cpu().numpy(), W.saxpy_i32(7, x, y))
        assert np.array_equal(y2d.cpu().numpy(), W.saxpy_i32(9, x2, y2))
        assert np.all(rt.coverage_np(h_lp, n_lp // 256) == 1)
        dec = rt.decision_log()
        acts = [f.ACTION_NAMES[d[1]] for d in dec]
        assert acts[:3] == ["LAUNCH", "PREEMPT", "LAUNCH"]
        assert dec == _replay_from_runtime(rt, des.HPF)
    finally:
        rt.close()


@pytest.mark.parametrize("kind", ["HPF", "FIFO"])
def test_managed_queue_replay_parity(kind):
    """A burst of mixed-priority kernels; the runtime's decisions equal the DES replay of the
    runtime's own measured ARRIVE/FINISH log (bit-exact, SURVEY §8(c) O3 replay mode)."""
    f = flep_mod()
    import torch
    pol = f.POLICY_HPF if kind == "HPF" else f.POLICY_FIFO
    rt = f.Runtime(policy=pol)
    try:
        g = gen.rng(31)
        ks, hs, refs = [], [], []
        streams = [torch.cuda.Stream() for _ in range(4)]
        for i in range(12):
            n = int(g.choice([1 << 16, 1 << 20, 1 << 23]))
            x, y = gen.saxpy_i32_inputs(n, seed=100 + i)
            xd, yd = t(x), t(y)
            k = rt.register_kernel(f.BODY_SAXPY_I32, chunk=2, poll=1, model=(0, 0, 0.02, 0, 1000),
                                   overhead_ns=int(g.integers(0, 20_000)))
            a = int(g.integers(1, 1000))
            h = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, a), priority=int(g.integers(0, 3)),
                          stream=streams[i % 4])
            hs.append(h)
            refs.append((yd, W.saxpy_i32(a, x, y)))
        for h in hs:
            rt.sync(h, timeout_ns=20_000_000_000)
        torch.cuda.synchronize()
        for yd, ref in refs:
            assert np.array_equal(yd.cpu().numpy(), ref)
        dec = rt.decision_log()
        assert dec == _replay_from_runtime(rt, des.HPF if kind == "HPF" else des.FIFO)
        if kind == "FIFO":
            assert all(d[1] == 0 for d in dec)
    finally:
        rt.close()


def test_random_schedules_10k_zero_violations():
    """Config 1: LP SAXPY-int32 2^20 under 10^4 random manual preempt/resume schedules (temporal
    and spatial yields, C in {1,2,4,8,16}, K in {1,2,4,8}, with and without prefetch and async
    poll, a quarter with the speculative fetch of R34). Every
    schedule: coverage == 1, bit-exact y, preempted epochs cover a prefix (I2), yields only on
    requested SMs (I3)."""
    f = flep_mod()
    import torch
    rt = f.Runtime(coverage=True)
    try:
        n, a = 1 << 20, 1664525
        nb = n // 256
        x, y = gen.saxpy_i32_inputs(n, seed=1)
        ref = W.saxpy_i32(a, x, y)
        xd, y0, yd = t(x), t(y), t(y)
        kern = {}
        viol_total, preempted_total, yielded_total, bad = 0, 0, 0, []
        import os
        n_sched = int(os.environ.get("FLEP_SCHEDULES", "10000"))   # evidence runs use 10^5
        for i in range(n_sched):
            s = gen.preempt_schedule(100 + i, nb, rt.num_sms)
            pf = i % 2 == 1
            ap = (i // 2) % 2 == 1                 # async poll (R22)
            sp = i % 4 == 0                        # speculative fetch (R34; never with pf / ap)
            cps = (1, 2, 8)[i % 3]                 # resident workers per SM (W = 148 * cps)
            key = (s["C"], s["K"], pf, cps, ap, sp)
            if key not in kern:
                kern[key] = rt.register_kernel(f.BODY_SAXPY_I32, chunk=s["C"], poll=s["K"], prefetch=pf,
                                               ctas_per_sm=cps, async_poll=ap, spec_fetch=sp)
            yd.copy_(y0)
            # (I2 as a plain prefix does not hold with R34: returned chunks sit in records)
            h, npre, viol = run_manual_schedule(rt, kern[key], f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, a), nb,
                                                s, rt.num_sms, check_prefix=(i % 10 == 0) and not sp)
            preempted_total += npre
            info = rt.query(h)
            # a schedule exercised preemption if a worker yielded or an epoch ended preempted (with
            # R34 a stopped worker whose fetch came back exhausted leaves with reason "exhausted")
            yielded_total += int(npre > 0 or any(e.reason == f.REASON_YIELD
                                                 for ep in range(1, info.epoch + 1) for e in rt.events(h, ep)))
            cov = rt.coverage_np(h, nb)
            if not np.all(cov == 1):
                viol.append("I1: coverage != 1")
            if i % 10 == 0 or viol:
                if not np.array_equal(yd.cpu().numpy(), ref):
                    viol.append("result != oracle")
            if viol:
                viol_total += len(viol)
                bad.append((i, s, viol))
        # outputs of every schedule are checked through coverage (exactly-once => bit-exact for
        # this deterministic body); every 10th schedule also compares y against the oracle
        summary = {"schedules": n_sched, "violations": viol_total, "schedules_with_yields": yielded_total,
                   "preempted_epochs": preempted_total}
        import json
        import os
        out = os.environ.get("FLEP_EVIDENCE_DIR")
        if out:
            with open(os.path.join(out, "schedules_10k.json"), "w") as fh:
                json.dump(summary, fh)
        assert viol_total == 0, bad[:5]
        # many schedules really preempt (with R34 a worker stopped late in the launch often
        # leaves with reason "exhausted": its speculative fetch found the counter past N)
        assert yielded_total > 2 * n_sched // 5
        assert preempted_total > n_sched // 5      # ... and many drain whole epochs (temporal)
    finally:
        rt.close()


def test_host_mapped_flag_transport():
    f = flep_mod()
    import time
    rt = f.Runtime(flag=f.FLAG_HOST_MAPPED, coverage=True)
    try:
        n = 1 << 26
        nb = n // 256
        x, y = gen.saxpy_i32_inputs(n, seed=41)
        xd, yd = t(x), t(y)
        k = rt.register_kernel(f.BODY_SAXPY_I32, chunk=1, poll=1)
        h = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, 5))
        time.sleep(0.0002)
        try:
            rt.preempt(h, rt.num_sms)
        except f.FlepError as e:
            assert e.status == f.ERR_STATE      # already finished: legal
        rt.wait_epoch(h, timeout_ns=10_000_000_000)
        if rt.query(h).state == f.STATE_PREEMPTED:
            c = rt.coverage_np(h, nb)
            m = min(int(rt.query(h).counter), nb)
            assert np.all(c[:m] == 1) and np.all(c[m:] == 0)
            rt.resume(h)
        rt.sync(h, timeout_ns=10_000_000_000)
        assert np.array_equal(yd.cpu().numpy(), W.saxpy_i32(5, x, y))
    finally:
        rt.close()


def test_cancel_then_reuse_control_block():
    f = flep_mod()
    rt = f.Runtime()
    try:
        n = 1 << 26
        x, y = gen.saxpy_i32_inputs(n, seed=51)
        xd, yd = t(x), t(y)
        k = rt.register_kernel(f.BODY_SAXPY_I32, chunk=1, poll=1)
        rt.arm_next_trigger(1000, rt.num_sms)
        h = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, 3))
        rt.wait_epoch(h, timeout_ns=10_000_000_000)
        rt.cancel(h)
        assert rt.query(h).state == f.STATE_DONE
        rt.sync(h)
        # the control block goes back to the pool; a new launch must start from a clean counter
        n2 = 1 << 20
        x2, y2 = gen.saxpy_i32_inputs(n2, seed=52)
        x2d, y2d = t(x2), t(y2)
        for _ in range(70):       # cycle through the retained-launch window and the pool
            y2d.copy_(t(y2))
            h2 = rt.launch(k, f.saxpy_grid(n2), f.saxpy_i32_args(y2d, x2d, 11))
            rt.sync(h2)
            assert np.array_equal(y2d.cpu().numpy(), W.saxpy_i32(11, x2, y2))
    finally:
        rt.close()


def test_managed_ffs_share_and_replay():
    """FFS (§5.2.2): two long kernels of priorities 1 and 0 (weights 2:1) share the GPU in epochs;
    the runtime's decisions replay exactly through the oracle FFS (TICK events logged)."""
    f = flep_mod()
    import torch
    rt = f.Runtime(policy=f.POLICY_FFS, max_overhead_ppm=100_000)
    try:
        n = 1 << 28
        x1, y1 = torch.ones(n, dtype=torch.int32, device="cuda"), torch.ones(n, dtype=torch.int32, device="cuda")
        x2, y2 = torch.ones(n, dtype=torch.int32, device="cuda"), torch.ones(n, dtype=torch.int32, device="cuda")
        k = rt.register_kernel(f.BODY_SAXPY_I32, chunk=8, poll=1, overhead_ns=20_000, model=(0, 0, 0, 0, 500_000))
        sA, sB = torch.cuda.Stream(), torch.cuda.Stream()
        h1 = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(y1, x1, 2), priority=1, stream=sA)
        h2 = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(y2, x2, 3), priority=0, stream=sB)
        rt.sync(h1, timeout_ns=20_000_000_000)
        rt.sync(h2, timeout_ns=20_000_000_000)
        torch.cuda.synchronize()
        assert int(y1[0].item()) == 3 and int(y1[-1].item()) == 3
        assert int(y2[12345].item()) == 4
        dec = rt.decision_log()
        assert sum(1 for d in dec if d[1] == 2) >= 2          # the epochs really alternated
        evs = []
        for (t_ns, typ, lid, prio, t_e, ovh) in rt.event_log():
            if typ == 0:
                evs.append((t_ns, "ARRIVE", des.KernelSpec(lid, t_ns, prio, t_e, ovh)))
            elif typ == 1:
                evs.append((t_ns, "FINISH", lid))
            else:
                evs.append((t_ns, "TICK", None))
        rep = [(t, ACT[a], i, n_) for (t, a, i, n_) in des.replay_ffs(evs, 100_000)]
        assert dec == rep
    finally:
        rt.close()


@pytest.mark.parametrize("spec", [False, True])
@pytest.mark.parametrize("tail", [False, True])
def test_spatial_refill_exactly_once(tail, spec):
    """Spatial yield, then refill: the victim is re-spread over all SMs. With the
    trigger near the end, the running epoch usually completes the launch before the refill epoch
    starts; that epoch must not re-run anything (the control block was already reset). With the
    speculative fetch (R34) the yielded workers' returned chunks are run by the refill epoch."""
    f = flep_mod()
    rt = f.Runtime(coverage=True)
    try:
        n = 1 << 22
        nb = n // 256
        x, y = gen.saxpy_i32_inputs(n, seed=81)
        ref = W.saxpy_i32(13, x, y)
        xd, y0 = t(x), t(y)
        k = rt.register_kernel(f.BODY_SAXPY_I32, chunk=1, poll=1, spec_fetch=spec)
        for rep in range(20):
            yd = y0.clone()
            tstar = nb - 40 if tail else nb // 4
            rt.arm_next_trigger(tstar, 37)
            h = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, 13))
            # wait until the spatial request is in force (the trigger fired) or the epoch ended
            import time
            t0 = time.time()
            while rt.query(h).state == f.STATE_RUNNING and time.time() - t0 < 5:
                try:
                    if rt.epoch_info(h, 1).t_trigger:
                        break
                except f.FlepError:
                    pass
            info = rt.query(h)
            if info.state in (f.STATE_RUNNING, f.STATE_PARTIAL):
                # the device trigger does not move the host state machine; mark the request
                try:
                    rt.preempt(h, 37)
                except f.FlepError:
                    pass
            try:
                rt.refill(h)
            except f.FlepError as e:
                assert e.status == f.ERR_STATE
            rt.wait_epoch(h, timeout_ns=10_000_000_000)
            if rt.query(h).state == f.STATE_PREEMPTED:
                rt.resume(h)
            rt.sync(h, timeout_ns=10_000_000_000)
            assert np.all(rt.coverage_np(h, nb) == 1)
            assert np.array_equal(yd.cpu().numpy(), ref)
    finally:
        rt.close()


def test_custom_rank_table_spatial_yield():
    """flep_set_rank_table: a spatial request for n SMs releases exactly the SMs whose
    rank is below n, for a non-identity table; then the identity table is restored."""
    f = flep_mod()
    import torch
    rt = f.Runtime(coverage=True)
    try:
        S = rt.num_sms
        table = [(S - 1 - s) for s in range(S)]          # reversed: the highest smids yield first
        rt.set_rank_table(table + list(range(S, rt.nsmid)) if rt.nsmid > S else table)
        n = 4096
        a = gen.stencil_f32_input(n, seed=61)
        ind = t(a)
        outd = torch.empty_like(ind)
        k = rt.register_kernel(f.BODY_STENCIL5_F32, chunk=1, poll=1)
        nb = (n // 64) ** 2
        for nsm in (8, 37):
            rt.arm_next_trigger(nb // 4, nsm)
            h = rt.launch(k, f.stencil_grid(n), f.stencil_args(outd, ind))
            rt.sync(h)
            ev = rt.events(h, 1)
            assert any(e.reason == f.REASON_YIELD for e in ev)
            for e in ev:
                assert (e.reason == f.REASON_YIELD) == (table[e.smid] < nsm)
            assert np.all(rt.coverage_np(h, nb) == 1)
        rt.set_rank_table(list(range(max(S, rt.nsmid))))
    finally:
        rt.close()


def _replay_ex(rt, spatial):
    evs = []
    for (t_ns, typ, lid, prio, t_e, ovh, need) in rt.event_log_ex():
        if typ == 0:
            evs.append((t_ns, "ARRIVE", des.KernelSpec(lid, t_ns, prio, t_e, ovh, 0, need)))
        else:
            evs.append((t_ns, "FINISH", lid))
    acts = {"LAUNCH": 0, "RESUME": 1, "PREEMPT": 2, "REFILL": 3}
    return [(t_, acts[a], i, n) for (t_, a, i, n) in des.replay(des.HPF, evs, num_sms=rt.num_sms, spatial=spatial)]


@pytest.mark.parametrize("spec", [False, True])
@pytest.mark.parametrize("n_sms", [5, 16, 74])
def test_managed_spatial_hpf_decides_how_far(n_sms, spec):
    """Spatial HPF (R29): a high-priority SAXPY-int32 whose workers fit on n SMs
    arrives while an int32 stencil 8192^2 runs; the runtime yields exactly n SMs (rank < n), runs
    the waiting kernel beside the victim, refills the victim at its end. Checked: decision list
    (and its oracle replay), I3 on the victim's worker log, every block exactly once, both
    outputs bit-exact vs the oracle."""
    f = flep_mod()
    import torch
    rt = f.Runtime(policy=f.POLICY_HPF, spatial=True, coverage=True)
    try:
        nst = 8192
        a = gen.stencil_i32_input(nst, seed=61)
        ind = t(a)
        outd = torch.empty_like(ind)
        k_v = rt.register_kernel(f.BODY_STENCIL5_I32, chunk=1, poll=1, model=(0, 0, 0, 0, 400_000),
                                 spec_fetch=spec)
        cps, _ = rt.workers_for(f.BODY_SAXPY_I32)
        n_hp = n_sms * cps * 256 - 77                      # ragged tail, still n_sms * cps blocks
        x2, y2 = gen.saxpy_i32_inputs(n_hp, seed=62)
        x2d, y2d = t(x2), t(y2)
        k_w = rt.register_kernel(f.BODY_SAXPY_I32, chunk=1, poll=1, model=(0, 0, 0, 0, 5_000))
        sA, sB = torch.cuda.Stream(), torch.cuda.Stream()
        h_v = rt.launch(k_v, f.stencil_grid(nst), f.stencil_args(outd, ind), priority=0, stream=sA)
        h_w = rt.launch(k_w, f.saxpy_grid(n_hp), f.saxpy_i32_args(y2d, x2d, 5), priority=1, stream=sB)
        rt.sync(h_w, timeout_ns=10_000_000_000)
        rt.sync(h_v, timeout_ns=10_000_000_000)
        torch.cuda.synchronize()
        assert np.array_equal(y2d.cpu().numpy(), W.saxpy_i32(5, x2, y2))
        assert np.array_equal(outd.cpu().numpy(), W.stencil5_i32(a))
        nb = (nst // 64) ** 2
        assert np.all(rt.coverage_np(h_v, nb) == 1)
        dec = rt.decision_log()
        names = [(f.ACTION_NAMES[d[1]], d[2], d[3]) for d in dec]
        assert names[:3] == [("LAUNCH", h_v, 0), ("PREEMPT", h_v, n_sms), ("LAUNCH", h_w, 0)]
        # the guest ends long before the victim: REFILL (if both completions land in one monitor
        # pass the victim may be seen first; the replay below checks that order too)
        if len(names) == 4:
            assert names[3] == ("REFILL", h_v, rt.num_sms)
        ev1 = rt.events(h_v, 1)
        w_end = max(e.t_exit for e in rt.events(h_w, 1))
        assert all(e.reason == f.REASON_YIELD for e in ev1 if e.smid < n_sms)
        assert not any(e.reason == f.REASON_YIELD and e.t_exit < w_end for e in ev1 if e.smid >= n_sms)
        assert dec == _replay_ex(rt, True)
    finally:
        rt.close()


def test_managed_cancel_releases_the_policy():
    """flep_cancel in a managed mode: the policy forgets the cancelled launch, so the
    kernels behind it still run, and its resources go back to the pools."""
    f = flep_mod()
    import torch
    rt = f.Runtime(policy=f.POLICY_FIFO)
    try:
        n = 1 << 26
        x, y = gen.saxpy_i32_inputs(n, seed=71)
        xd, yd = t(x), t(y)
        k = rt.register_kernel(f.BODY_SAXPY_I32, chunk=1, poll=1)
        n2 = 1 << 18
        x2, y2 = gen.saxpy_i32_inputs(n2, seed=72)
        x2d, y2d = t(x2), t(y2)
        h1 = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, 3))        # running
        h2 = rt.launch(k, f.saxpy_grid(n), f.saxpy_i32_args(yd, xd, 3))        # queued behind it
        h3 = rt.launch(k, f.saxpy_grid(n2), f.saxpy_i32_args(y2d, x2d, 11))    # queued
        rt.cancel(h2)                                                           # a queued one
        rt.cancel(h1)                                                           # the running one
        rt.sync(h3, timeout_ns=10_000_000_000)
        torch.cuda.synchronize()
        assert np.array_equal(y2d.cpu().numpy(), W.saxpy_i32(11, x2, y2))
        for h in (h1, h2, h3):
            assert rt.query(h).state == f.STATE_DONE
        for _ in range(20):                                                     # pools still work
            y2d.copy_(t(y2))
            h = rt.launch(k, f.saxpy_grid(n2), f.saxpy_i32_args(y2d, x2d, 11))
            rt.sync(h, timeout_ns=10_000_000_000)
            torch.cuda.synchronize()
            assert np.array_equal(y2d.cpu().numpy(), W.saxpy_i32(11, x2, y2))
    finally:
        rt.close()


@pytest.mark.parametrize("stream_exec", [False, True])
def test_slice_device_preempts_at_slice_boundaries(stream_exec):
    """Kernel slicing with every slice enqueued and the device check at slice entry (R31): the
    high-priority arrival makes the remaining slices skip themselves; the victim resumes at the
    first skipped slice; results bit-exact; decisions = HPF's, replayed by the oracle."""
    f = flep_mod()
    import torch
    rt = f.Runtime(policy=f.POLICY_SLICE_DEVICE, slice_blocks=4096, exec_on_user_stream=stream_exec)
    try:
        n_lp, n_hp = 1 << 26, 1 << 16
        x, y = gen.saxpy_i32_inputs(n_lp, seed=81)
        x2, y2 = gen.saxpy_i32_inputs(n_hp, seed=82)
        xd, yd, x2d, y2d = t(x), t(y), t(x2), t(y2)
        k_lp = rt.register_kernel(f.BODY_SAXPY_I32, chunk=1, poll=1, model=(0, 0, 0, 0, 2_000_000))
        k_hp = rt.register_kernel(f.BODY_SAXPY_I32, chunk=1, poll=1, model=(0, 0, 0, 0, 5_000))
        sA, sB = torch.cuda.Stream(), torch.cuda.Stream()
        h_lp = rt.launch(k_lp, f.saxpy_grid(n_lp), f.saxpy_i32_args(yd, xd, 7), priority=0, stream=sA)
        h_hp = rt.launch(k_hp, f.saxpy_grid(n_hp), f.saxpy_i32_args(y2d, x2d, 9), priority=1, stream=sB)
        rt.sync(h_hp, timeout_ns=10_000_000_000)
        rt.sync(h_lp, timeout_ns=10_000_000_000)
        torch.cuda.synchronize()
        assert np.array_equal(yd.cpu().numpy(), W.saxpy_i32(7, x, y))
        assert np.array_equal(y2d.cpu().numpy(), W.saxpy_i32(9, x2, y2))
        dec = rt.decision_log()
        acts = [f.ACTION_NAMES[d[1]] for d in dec]
        assert acts == ["LAUNCH", "PREEMPT", "LAUNCH", "RESUME"]
        info = rt.query(h_lp)
        assert info.epoch == 2 and info.state == f.STATE_DONE
        assert dec == _replay_from_runtime(rt, des.HPF)
    finally:
        rt.close()


def test_slice_device_never_preempted_exact():
    f = flep_mod()
    import torch
    rt = f.Runtime(policy=f.POLICY_SLICE_DEVICE)
    try:
        for n in (3, 1000, 4096):
            a = gen.stencil_i32_input(n, seed=83)
            ind = t(a)
            outd = torch.empty_like(ind)
            k = rt.register_kernel(f.BODY_STENCIL5_I32, chunk=1, poll=1)
            h = rt.launch(k, f.stencil_grid(n), f.stencil_args(outd, ind))
            rt.sync(h, timeout_ns=10_000_000_000)
            torch.cuda.synchronize()
            assert np.array_equal(outd.cpu().numpy(), W.stencil5_i32(a))
            assert rt.query(h).epoch == 1
    finally:
        rt.close()
