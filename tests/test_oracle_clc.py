"""Pins for oracle/clc.py (R25, the CLC task fetch): exhaustive interleavings of the
hardware's launch/cancel choices, the workers' steps and preempt/resume requests on Fig. 2's
2-SM case, exactly-once coverage at the end of every run, including runs where the request
is never withdrawn, and a planted bug the checker must catch."""
import itertools

import pytest

from oracle import clc


def _cfg(**kw):
    base = dict(n_blocks=5, chunk=1, poll=1, slot_sm=(0, 1), num_sms=2, preempt_widths=(1, 2),
                max_events=2)
    base.update(kw)
    return clc.Config(**base)


@pytest.mark.parametrize("C,K", list(itertools.product([1, 2], [1, 2])))
def test_exhaustive_exactly_once(C, K):
    r = clc.explore(_cfg(n_blocks=4 if C == 1 else 5, chunk=C, poll=K))
    assert r.violations == set()
    assert r.terminals > 0 and r.yields_seen > 0      # requests really made workers leave


def test_request_never_withdrawn_still_completes():
    # without resume events, queued CTAs still start (the hardware launches them into the freed
    # slots), run their own chunk and leave: the launch completes, every block once
    r = clc.explore(_cfg(n_blocks=4, allow_resume=False, max_events=1, preempt_widths=(2,)))
    assert r.violations == set()
    assert r.yields_seen > 0


def test_more_slots_than_chunks_and_ragged_chunk():
    r = clc.explore(_cfg(n_blocks=5, chunk=2, slot_sm=(0, 0, 1, 1), preempt_widths=(1,), max_events=2))
    assert r.violations == set()


def test_planted_drop_claimed_chunk_is_caught():
    r = clc.explore(_cfg(n_blocks=4, bug_drop_claimed_on_stop=True))
    assert any("liveness" in v for v in r.violations)


def test_hand_traced_cancel_then_yield():
    # one slot on SM0, N = 3, C = K = 1: launch CTA 0, poll, cancel CTA 1, run 0, request,
    # poll -> stop, run 1 and leave; CTA 2 is still queued and starts in the freed slot
    cfg = clc.Config(n_blocks=3, chunk=1, poll=1, slot_sm=(0,), num_sms=2, preempt_widths=(2,),
                     max_events=1, allow_resume=False)
    st = clc.initial_state(cfg)
    for lab in ["s0.launch0", "s0.poll", "s0.cancel1", "s0.run", "preempt(2)", "s0.poll_stop",
                "s0.run_leave", "s0.launch2", "s0.poll_stop", "s0.run_leave"]:
        st = dict(clc.successors(cfg, st))[lab]
    queue, slots, cov, req, ev, ylog = st
    assert cov == (1, 1, 1) and not queue and slots[0][0] == clc.FREE
    assert [y[1] for y in ylog] == [clc.R_YIELD, clc.R_YIELD]
