"""Pins for the FFS policy of oracle/des.py (§5.2.2; Figs. 13-14)."""
from oracle import des


def test_t_min_closed_form():
    p = des.FfsPolicy(max_overhead_ppm=100_000)
    p.on_arrival(0, des.KernelSpec(0, 0, 1, 10**9, 20_000, 10**9))
    p.on_arrival(1, des.KernelSpec(1, 1, 0, 10**9, 10_000, 10**9))
    # sum O / (T sum W) <= 0.1  ->  T >= 30000 / (0.1 * 3) = 100000 ns
    assert p.t_min() == 100_000


def test_weighted_share_two_to_one():
    # two never-ending kernels, priorities 1 and 0 -> weights 2:1 -> GPU shares 2/3 and 1/3
    ks = [des.KernelSpec(0, 0, 1, 10**12, 20_000, 10**12), des.KernelSpec(1, 0, 0, 10**12, 20_000, 10**12)]
    r = des.simulate_ffs(ks, 100_000, des.SimParams(), horizon_ns=50_000_000)
    share = r.busy[0] / (r.busy[0] + r.busy[1])
    assert abs(share - 2 / 3) < 0.01


def test_overhead_fraction_equals_max_overhead():
    # when each preemption really costs its estimate O (drain = O, no useful progress assumed
    # lost), the time spent switching per round is sum O / (T sum W) = max_overhead (Fig. 14)
    O = 50_000
    ks = [des.KernelSpec(0, 0, 1, 10**12, O, 10**12), des.KernelSpec(1, 0, 0, 10**12, O, 10**12)]
    p = des.FfsPolicy(100_000)
    for k in ks:
        p.on_arrival(0, k)
    T = p.t_min()
    round_len = T * (2 + 1)
    assert abs(2 * O / round_len - 0.10) < 1e-3


def test_lone_kernel_is_never_preempted():
    ks = [des.KernelSpec(0, 0, 0, 5_000_000, 10_000, 5_000_000)]
    r = des.simulate_ffs(ks, 100_000)
    assert [d[1] for d in r.decisions] == ["LAUNCH"]
    assert r.finish[0] == 5_000_000


def test_round_order_and_replay():
    ks = [des.KernelSpec(0, 0, 0, 3_000_000, 10_000, 3_000_000),
          des.KernelSpec(1, 100, 2, 2_000_000, 10_000, 2_000_000),
          des.KernelSpec(2, 200, 1, 1_000_000, 10_000, 1_000_000)]
    r = des.simulate_ffs(ks, 100_000, des.SimParams(drain_ns=2_000, start_ns=3_000))
    assert set(r.finish) == {0, 1, 2}
    assert des.replay_ffs(r.events, 100_000) == r.decisions
    # kernels 1 and 2 arrive during kernel 0's first epoch and join the end of that round
    runs = [d[2] for d in r.decisions if d[1] in ("LAUNCH", "RESUME")]
    assert runs[:3] == [0, 1, 2]
    # next round: priority descending (1: prio 2, 2: prio 1, 0: prio 0)
    assert runs[3:6] == [1, 2, 0]
