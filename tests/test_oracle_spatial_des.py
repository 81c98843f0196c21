"""Pins of the spatial HPF policy and its simulate mode (oracle/des.py Policy(spatial=True),
simulate_rates; R29 = SURVEY A9/A13/A15).

What fixes them independently of the code under test:
  * spatial decisions switched off reduce simulate_rates to the temporal simulate() (the paper's
    Fig. 6 as printed), on random traces with drain and start delays;
  * a waiting kernel that needs every SM (or declares no need) is a temporal preemption;
  * closed forms of a two-kernel co-run: the victim loses exactly the work of the n released
    SMs for the guest's duration (T_v + T_g * n / S), the guest runs as if alone;
  * the T_r bookkeeping of a spatially sharing victim (A13) by hand;
  * hand-traced decision lists for arrivals during a co-run and for the victim finishing first.
"""
import pytest

from oracle import des
from synth import gen

S = 148


def _ks(i, arr, prio, t_true, need=0, t_e=None, o=0):
    return des.KernelSpec(i, arr, prio, t_true if t_e is None else t_e, o, t_true, need)


def _random(seed, n=30, need_max=148):
    g = gen.rng(seed)
    ks, t = [], 0
    for i in range(n):
        t += int(g.integers(0, 300_000))
        true = int(g.integers(1_000, 2_000_000))
        est = max(1, int(true * g.uniform(0.6, 1.4)))
        ks.append(_ks(i, t, int(g.integers(0, 3)), true, int(g.integers(0, need_max + 1)), est,
                      int(g.integers(0, 50_000))))
    return ks


@pytest.mark.parametrize("seed", range(15))
def test_rates_engine_without_spatial_equals_temporal_simulate(seed):
    ks = _random(seed)
    p = des.SimParams(drain_ns=seed * 900, start_ns=2_000 + seed * 100)
    a = des.simulate(des.HPF, ks, p)
    b = des.simulate_rates(ks, p, spatial=False)
    assert a.decisions == b.decisions
    assert a.finish == b.finish
    assert a.events == b.events


@pytest.mark.parametrize("need", [0, S, S + 10])
def test_guest_needing_every_sm_is_temporal(need):
    ks = [_ks(0, 0, 0, 1_000_000), _ks(1, 100_000, 1, 50_000, need)]
    a = des.simulate(des.HPF, ks)
    b = des.simulate_rates(ks, spatial=True)
    assert a.decisions == b.decisions and a.finish == b.finish
    assert all(d[1] != "REFILL" for d in b.decisions)


@pytest.mark.parametrize("n", [1, 5, 8, 37, 74, 147])
def test_two_kernel_corun_closed_form(n):
    tv, tg, a = 3_000_000, S * 1_000, 400_000          # tg multiple of S: exact shares
    ks = [_ks(0, 0, 0, tv), _ks(1, a, 1, tg, n)]
    r = des.simulate_rates(ks, spatial=True)
    assert r.decisions == [(0, "LAUNCH", 0, 0), (a, "PREEMPT", 0, n), (a, "LAUNCH", 1, 0),
                           (a + tg, "REFILL", 0, S)]
    assert r.finish[1] == a + tg                         # the guest runs as if alone
    assert r.finish[0] == tv + tg * n // S               # the victim loses n/S of tg
    assert r.turnaround[1] == tg


def test_two_kernel_corun_with_drain_and_start_delays():
    tv, tg, a, d, s = 3_000_000, S * 2_000, 500_000, 7_400, 3_000
    n = 10
    ks = [_ks(0, 0, 0, tv), _ks(1, a, 1, tg, n)]
    r = des.simulate_rates(ks, des.SimParams(drain_ns=d, start_ns=s), spatial=True)
    g_start = a + d + s
    assert r.finish[1] == g_start + tg
    # victim: full rate on [s, a + d], (S - n)/S on [a + d, G end], stopped for s, full after
    done = (a + d - s) + (g_start + tg - (a + d)) * (S - n) // S
    assert r.finish[0] == g_start + tg + s + (tv - done)


def test_victim_t_r_falls_at_the_held_share():
    pol = des.Policy(des.HPF, S, spatial=True)
    pol.on_arrival(0, _ks(0, 0, 0, 1_000_000))
    pol.on_arrival(200_000, _ks(1, 200_000, 1, 50_000, 20))
    pol.on_finish(200_000 + 74_000, 1)
    # at the guest's finish: 1e6 - 2e5 (alone) - floor(74000 * 128 / 148)
    assert pol.k[0].t_r == 1_000_000 - 200_000 - 74_000 * (S - 20) // S
    assert pol.decisions[-1] == (274_000, "REFILL", 0, S)
    assert pol.running == 0 and pol.guest is None


def test_arrivals_during_corun_wait_then_outrank_the_victim():
    pol = des.Policy(des.HPF, S, spatial=True)
    pol.on_arrival(0, _ks(0, 0, 0, 5_000_000))
    pol.on_arrival(10, _ks(1, 10, 2, 100_000, 8))        # guest, 8 SMs
    pol.on_arrival(20, _ks(2, 20, 3, 100_000, 16))       # outranks everyone: waits for the guest
    pol.on_arrival(30, _ks(3, 30, 0, 10, 1))             # equal to the victim: waits
    assert pol.decisions == [(0, "LAUNCH", 0, 0), (10, "PREEMPT", 0, 8), (10, "LAUNCH", 1, 0)]
    pol.on_finish(100_010, 1)
    # refill, then the waiting prio-3 kernel is a case-1 arrival against the victim (16 SMs)
    assert pol.decisions[3:] == [(100_010, "REFILL", 0, S), (100_010, "PREEMPT", 0, 16),
                                 (100_010, "LAUNCH", 2, 0)]
    assert pol.guest == 2 and pol.running == 0
    pol.on_finish(200_010, 2)
    # refill; kernel 3 (T_r 10) vs the victim (T_r large) at equal priority: SRPT preempts it
    assert pol.decisions[6:] == [(200_010, "REFILL", 0, S), (200_010, "PREEMPT", 0, S),
                                 (200_010, "LAUNCH", 3, 0)]
    pol.on_finish(200_020, 3)
    assert pol.decisions[-1] == (200_020, "RESUME", 0, 0)


def test_victim_finishing_first_promotes_the_guest():
    ks = [_ks(0, 0, 0, 100_000), _ks(1, 90_000, 1, 5_000_000, 30), _ks(2, 95_000, 0, 1_000, 2)]
    r = des.simulate_rates(ks, spatial=True)
    # the victim has 10 us of work left at 118/148 of full speed: done at 90000 + ceil(10000*148/118)
    assert r.finish[0] == 90_000 + -(-10_000 * S // (S - 30))
    # kernel 2 waited (arrival during the co-run); after the victim the guest runs alone and
    # kernel 2 (lower priority than the guest) stays queued until the guest is done
    assert r.decisions == [(0, "LAUNCH", 0, 0), (90_000, "PREEMPT", 0, 30), (90_000, "LAUNCH", 1, 0),
                           (5_090_000, "LAUNCH", 2, 0)]
    assert r.finish[1] == 5_090_000 and r.finish[2] == 5_091_000


def test_spatial_width_feeds_the_decision():
    # a kernel of 40 CTAs at 8 CTAs per SM needs 5 SMs -> PREEMPT(victim, 5)
    n = des.spatial_width(40, 8, S)
    ks = [_ks(0, 0, 0, 1_000_000), _ks(1, 10, 1, 1_000, n)]
    r = des.simulate_rates(ks, spatial=True)
    assert (10, "PREEMPT", 0, 5) in r.decisions


@pytest.mark.parametrize("seed", range(10))
def test_replay_reproduces_simulate_rates(seed):
    ks = _random(seed, need_max=60)
    r = des.simulate_rates(ks, des.SimParams(drain_ns=3_000, start_ns=2_000), spatial=True)
    assert des.replay(des.HPF, r.events, spatial=True) == r.decisions
    assert sorted(r.finish) == [k.id for k in ks]            # every kernel finishes once
    # a REFILL only ever follows a spatial PREEMPT of the same kernel (one co-run at a time)
    partial = None
    for (t, act, kid, n) in r.decisions:
        if act == "PREEMPT" and n < S:
            assert partial is None or partial not in r.finish or r.finish[partial] <= t
            partial = kid
        elif act == "REFILL":
            assert kid == partial
            partial = None
