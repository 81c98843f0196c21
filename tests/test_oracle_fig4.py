"""The plain Fig. 4 model (oracle/fig4.py) and its agreement with the B200 worker model
(oracle/coverage.py) restricted to the paper's configuration (C = K = 1, no static first chunk,
no prefetch, no async poll: DESIGN.md R20-R23 switched off) — VERDICT r1 #7.

Pins of the plain model itself: exhaustive interleavings on Fig. 2's 2-SM x 2-CTA case
find no violation of I1-I3 and every run completes; the counter ends at N + (failing pulls), a
closed form for uninterrupted runs; a planted "check the flag between pull and process" bug is
caught (the dropped task is never run: I2 and liveness fail)."""
import pytest

from oracle import coverage as full
from oracle import fig4


def _collect_full(cfg):
    """(epoch, cov, ctr) of every drained preempted epoch and the completion counters of the full
    model, by exhaustive DFS (the same reachable states as coverage.explore)."""
    start = full.initial_state(cfg)
    seen, stack = {start}, [start]
    drained, finals = set(), set()
    while stack:
        st = stack.pop()
        ctr, ctrl, done, yields, cov, epoch, status, workers, ev, extra = st
        if status == full.ST_PREEMPTED and full._all_gone(workers):
            drained.add((epoch, cov, ctr))
        nxt = full.successors(cfg, st)
        if not nxt:
            finals.add(extra[2] if extra[1] else ctr)
        for _, s2 in nxt:
            if s2 not in seen:
                seen.add(s2)
                stack.append(s2)
    return drained, finals


CASES = [
    # (N, worker SMs, widths, events)
    (3, (0, 0, 1, 1), (2,), 1),
    (4, (0, 0, 1, 1), (1, 2), 2),
    (5, (0, 1), (1, 2), 2),
    (4, (0, 1, 1), (1, 2), 2),
]


@pytest.mark.parametrize("n,sms,widths,events", CASES)
def test_plain_fig4_invariants(n, sms, widths, events):
    r = fig4.explore(fig4.Fig4Config(n, sms, 2, widths, events))
    assert not r.violations, r.violations
    assert r.drained                                   # preempted epochs do happen
    assert all(n <= c <= n + len(sms) for c in r.final_counters)


@pytest.mark.parametrize("n,w", [(1, 1), (3, 2), (5, 4)])
def test_plain_fig4_uninterrupted_counter_closed_form(n, w):
    r = fig4.explore(fig4.Fig4Config(n, tuple(i % 2 for i in range(w)), 2, (), 0))
    assert r.final_counters == {n + w}                 # N pulls that found work + one failing pull each
    assert not r.drained


def test_plain_fig4_catches_planted_bug():
    r = fig4.explore(fig4.Fig4Config(3, (0, 0, 1, 1), 2, (1, 2), 2, bug_check_after_pull=True))
    assert any("I2" in v for v in r.violations)
    assert any("liveness" in v for v in r.violations)


@pytest.mark.parametrize("n,sms,widths,events", CASES)
def test_full_model_restricted_to_fig4_reaches_the_same_outcomes(n, sms, widths, events):
    """The B200 worker model with its refinements switched off and the plain Fig. 4 model drain
    the same preempted epochs (same coverage, same counter, in the same epoch) and complete with
    the same counters, over every interleaving."""
    plain = fig4.explore(fig4.Fig4Config(n, sms, 2, widths, events))
    cfg = full.Config(n_blocks=n, chunk=1, poll=1, worker_sm=sms, num_sms=2, preempt_widths=widths,
                      max_events=events)
    drained, finals = _collect_full(cfg)
    assert drained == plain.drained
    assert finals == plain.final_counters
