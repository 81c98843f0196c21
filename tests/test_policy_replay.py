"""Replay parity: the C++ decision engine inside libflep.so (flep_policy_*) must reproduce the
oracle DES's decision list bit for bit on the same event traces (BJ "the
scheduler's decision sequence" bit-exact). Host only — no GPU."""
import pytest

from oracle import des
from synth import gen


@pytest.fixture(scope="module")
def flep():
    from paper_conf_asplos_wulzj17_b200 import build, flep as F
    build.build()
    return F


ACT = {"LAUNCH": 0, "RESUME": 1, "PREEMPT": 2, "REFILL": 3}
KIND = {des.FIFO: 1, des.HPF: 2, des.SLICE: 3, des.REORDER: 5}


def replay_cpp(F, kind, events, spatial=False):
    p = F.PolicyEngine(KIND[kind], spatial=spatial)
    for ev in events:
        if ev[1] == "ARRIVE":
            s = ev[2]
            p.arrive(ev[0], s.id, s.priority, s.t_e, s.overhead, s.sms_need)
        else:
            p.finish(ev[0], ev[2])
    return p.decisions()


def as_tuples(dec):
    return [(t, ACT[a], i, n) for (t, a, i, n) in dec]


def random_trace(seed, n, prios=3, tight=False):
    g = gen.rng(seed)
    ks, t = [], 0
    for i in range(n):
        t += int(g.integers(0, 50_000 if tight else 400_000))
        true = int(g.integers(1_000, 2_000_000))
        est = max(1, int(true * g.uniform(0.5, 1.5)))
        ks.append(des.KernelSpec(i, t, int(g.integers(0, prios)), est, int(g.integers(0, 80_000)), true))
    return ks


@pytest.mark.parametrize("kind", [des.FIFO, des.HPF, des.SLICE, des.REORDER])
@pytest.mark.parametrize("seed", range(25))
def test_replay_parity_random_traces(flep, kind, seed):
    ks = random_trace(seed, 40, prios=1 + seed % 4, tight=seed % 2 == 0)
    params = des.SimParams(drain_ns=int(seed * 700), start_ns=3_000,
                           slice_ns=150_000 if kind == des.SLICE else 0, slice_gap_ns=6_000)
    sim = des.simulate(kind, ks, params)
    assert as_tuples(sim.decisions) == replay_cpp(flep, kind, sim.events)


@pytest.mark.parametrize("seed", range(25))
def test_replay_parity_spatial_hpf(flep, seed):
    """Spatial HPF (R29): decision lists with n_sms < 148 and REFILLs replay bit-exactly."""
    g = gen.rng(500 + seed)
    ks = random_trace(seed, 40, prios=1 + seed % 4, tight=seed % 2 == 0)
    for k in ks:
        k.sms_need = int(g.integers(0, 160))
    sim = des.simulate_rates(ks, des.SimParams(drain_ns=seed * 500, start_ns=2_500), spatial=True)
    assert as_tuples(sim.decisions) == replay_cpp(flep, des.HPF, sim.events, spatial=True)


def test_replay_parity_spatial_hand_trace(flep):
    ks = [des.KernelSpec(0, 0, 0, 5_000_000, 0, 5_000_000, 0),
          des.KernelSpec(1, 10, 2, 100_000, 0, 100_000, 8),
          des.KernelSpec(2, 20, 3, 100_000, 0, 100_000, 16),
          des.KernelSpec(3, 30, 0, 10, 0, 10, 1)]
    sim = des.simulate_rates(ks, spatial=True)
    assert sum(1 for d in sim.decisions if d[1] == "REFILL") == 2
    assert as_tuples(sim.decisions) == replay_cpp(flep, des.HPF, sim.events, spatial=True)


def test_replay_parity_table1_pairs(flep):
    T = {"CFD": (11106, 521), "NN": (15775, 728), "PF": (7364, 811), "PL": (5419, 952),
         "MD": (15905, 938), "SPMV": (5840, 484), "MM": (2579, 1499), "VA": (30634, 720)}
    for lp in T:
        for hp in T:
            if lp == hp:
                continue
            for prio_hp in (0, 1):
                ks = [des.KernelSpec(0, 0, 0, T[lp][0] * 1000, 500, T[lp][0] * 1000),
                      des.KernelSpec(1, 1, prio_hp, T[hp][1] * 1000, 500, T[hp][1] * 1000)]
                sim = des.simulate(des.HPF, ks)
                assert as_tuples(sim.decisions) == replay_cpp(flep, des.HPF, sim.events)


def test_ties_and_equal_arrivals(flep):
    # identical T_r and arrival times: arrival order decides (A14)
    ks = [des.KernelSpec(i, 1000 * (i // 3), 0, 5000, 0, 5000) for i in range(9)]
    sim = des.simulate(des.HPF, ks)
    assert as_tuples(sim.decisions) == replay_cpp(flep, des.HPF, sim.events)
    order = [d[2] for d in sim.decisions if d[1] in ("LAUNCH", "RESUME")]
    assert order == sorted(order)


@pytest.mark.parametrize("seed", range(12))
def test_ffs_replay_parity(flep, seed):
    g = gen.rng(500 + seed)
    ks, t = [], 0
    for i in range(int(g.integers(2, 9))):
        t += int(g.integers(0, 3_000_000))
        true = int(g.integers(100_000, 20_000_000))
        ks.append(des.KernelSpec(i, t, int(g.integers(0, 3)), true, int(g.integers(1_000, 200_000)), true))
    ppm = int(g.choice([50_000, 100_000, 200_000]))
    sim = des.simulate_ffs(ks, ppm, des.SimParams(drain_ns=int(g.integers(0, 20_000)), start_ns=5_000))
    p = flep.PolicyEngine(4)
    p.set_max_overhead(ppm)
    for ev in sim.events:
        if ev[1] == "ARRIVE":
            s = ev[2]
            p.arrive(ev[0], s.id, s.priority, s.t_e, s.overhead)
        elif ev[1] == "FINISH":
            p.finish(ev[0], ev[2])
        else:
            assert p.tick(ev[0])
    assert as_tuples(sim.decisions) == p.decisions()
    assert len(sim.finish) == len(ks)


def test_b200_queue_trace_replays_exactly_through_the_oracle():
    """The runtime's own event log of the configs[3] queue run on the B200 (64 kernels, FIFO,
    FLEP-HPF and REORDER; tests/golden/queue_logs_r01.json, written by bench.py --config queue
    with FLEP_EVIDENCE_DIR) replayed through the oracle DES gives the runtime's decision list bit
    for bit (SURVEY §8(c) O3 replay mode)."""
    import json
    import os
    path = os.path.join(os.path.dirname(__file__), "golden", "queue_logs_r01.json")
    with open(path) as fh:
        logs = json.load(fh)["logs"]
    kinds = {"FIFO": des.FIFO, "HPF": des.HPF, "REORDER": des.REORDER}
    checked = 0
    for name, kind in kinds.items():
        evl, dec = logs[name]["events"], logs[name]["decisions"]
        evs = [(t, "ARRIVE", des.KernelSpec(i, t, p, te, o)) if ty == 0 else (t, "FINISH", i)
               for (t, ty, i, p, te, o) in evl]
        assert as_tuples(des.replay(kind, evs)) == [tuple(d) for d in dec], name
        checked += len(dec)
    assert checked > 100
    assert sum(1 for d in logs["HPF"]["decisions"] if d[1] == ACT["PREEMPT"]) > 5


def test_b200_slice_queue_log_replays_exactly():
    """Round-2 B200 queue run (configs[3], tests/golden/queue_logs_r02.json): every policy's log,
    including kernel slicing (SLICE takes HPF's decisions, R16), replays bit for bit."""
    import json
    import os
    path = os.path.join(os.path.dirname(__file__), "golden", "queue_logs_r02.json")
    with open(path) as fh:
        logs = json.load(fh)["logs"]
    kinds = {"FIFO": des.FIFO, "HPF": des.HPF, "SLICE": des.SLICE, "REORDER": des.REORDER}
    for name, kind in kinds.items():
        evl, dec = logs[name]["events"], logs[name]["decisions"]
        evs = [(t, "ARRIVE", des.KernelSpec(i, t, p, te, o)) if ty == 0 else (t, "FINISH", i)
               for (t, ty, i, p, te, o) in evl]
        assert as_tuples(des.replay(kind, evs)) == [tuple(d) for d in dec], name
    assert sum(1 for d in logs["SLICE"]["decisions"] if d[1] == ACT["PREEMPT"]) > 0


def test_b200_managed_spatial_log_replays_exactly():
    """The managed spatial-HPF run of configs[2] on the B200 (tests/golden/spatial_managed_logs_r02.json,
    written by bench.py --config spatial_managed): the runtime's event log (with each launch's
    sms_need) replayed through the oracle DES with spatial decisions gives its decision list bit
    for bit, including PREEMPT widths 8/16/32/74 (< 148) and the REFILLs (R29)."""
    import json
    import os
    path = os.path.join(os.path.dirname(__file__), "golden", "spatial_managed_logs_r02.json")
    with open(path) as fh:
        d = json.load(fh)
    evs = [(t, "ARRIVE", des.KernelSpec(i, t, p, te, o, 0, need)) if ty == 0 else (t, "FINISH", i)
           for (t, ty, i, p, te, o, need) in d["events"]]
    got = as_tuples(des.replay(des.HPF, evs, num_sms=d["num_sms"], spatial=True))
    assert got == [tuple(x) for x in d["decisions"]]
    widths = sorted({x[3] for x in d["decisions"] if x[1] == ACT["PREEMPT"]})
    assert widths == [8, 16, 32, 74, 148]
    assert sum(1 for x in d["decisions"] if x[1] == ACT["REFILL"]) >= 40


def test_b200_corun_matrix_logs_replay_exactly():
    """The co-run matrices on the B200 (bench.py --config coruns: E4 high-priority pairs, E6
    equal-priority pairs, E8 triplets, Figs. 8 / 10 / 12; tests/golden/corun_logs_r02.json): every
    case's event log under FIFO, FLEP-HPF and REORDER replayed through the oracle DES gives the
    runtime's decision list bit for bit; every HPF case preempts its large first kernel."""
    import json
    import os
    path = os.path.join(os.path.dirname(__file__), "golden", "corun_logs_r02.json")
    with open(path) as fh:
        logs = json.load(fh)["logs"]
    kinds = {"FIFO": des.FIFO, "HPF": des.HPF, "REORDER": des.REORDER}
    seen = {"E4": 0, "E6": 0, "E8": 0}
    for key, lg in logs.items():
        exp, case, pol = key.split("/")
        evs = [(t, "ARRIVE", des.KernelSpec(i, t, p, te, o)) if ty == 0 else (t, "FINISH", i)
               for (t, ty, i, p, te, o) in lg["events"]]
        assert as_tuples(des.replay(kinds[pol], evs)) == [tuple(d) for d in lg["decisions"]], key
        if pol == "HPF":
            seen[exp] += 1
            assert any(d[1] == ACT["PREEMPT"] for d in lg["decisions"]), key
    assert seen == {"E4": 16, "E6": 16, "E8": 28}
