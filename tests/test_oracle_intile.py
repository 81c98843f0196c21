"""Pins for oracle/intile.py (in-tile preemption; R21): exhaustive
interleavings of k-steps, in-tile and block-boundary polls, preempt and resume on tiny cases
(two SMs, as Fig. 2), two planted protocol bugs the checker must catch, and the
uninterrupted closed form."""
import pytest

from oracle import intile as it


def _cfg(**kw):
    base = dict(n_blocks=3, chunk=1, poll=1, k_steps=3, kpoll=1, worker_sm=(0, 1), num_sms=2,
                preempt_widths=(1, 2), max_events=2)
    base.update(kw)
    return it.Config(**base)


@pytest.mark.parametrize("kw", [
    dict(),                                                  # C = 1, poll every k-step
    dict(chunk=2, n_blocks=4, k_steps=2),                    # rest of the chunk rides in the record
    dict(kpoll=2, k_steps=4),                                # poll every 2 k-steps
    dict(poll=2, n_blocks=4, k_steps=2),                     # block-boundary poll every 2 chunks
    dict(min_left=1),                                        # finish when <= 1 k-step is left
    dict(worker_sm=(0, 0, 1), n_blocks=4, k_steps=2),        # two workers on one SM
    dict(preempt_widths=(2,), max_events=3, n_blocks=4, k_steps=2),   # repeated temporal yields
])
def test_exhaustive_no_violations(kw):
    r = it.explore(_cfg(**kw))
    assert r.violations == set()
    assert r.preempted_epoch_ends > 0
    assert r.intile_yields > 0          # workers really stop inside blocks


def test_planted_restore_from_zero_is_caught():
    # a resume that restarts the block's k-loop at 0 double-accumulates (J1)
    r = it.explore(_cfg(bug_restore_from_zero=True))
    assert any(v.startswith("J1") for v in r.violations)


def test_planted_dropped_chunk_rest_is_caught():
    # a record that forgets the unstarted blocks of its chunk loses them (liveness)
    r = it.explore(_cfg(chunk=2, n_blocks=4, k_steps=2, bug_drop_chunk_rest=True))
    assert any(v.startswith("liveness") for v in r.violations)


@pytest.mark.parametrize("n,C,ws", [(3, 1, (0, 1)), (5, 2, (0, 1)), (1, 1, (0, 1)), (4, 3, (0,))])
def test_uninterrupted_closed_form(n, C, ws):
    # without requests every block is accumulated K times and written once; the counter ends at
    # W*C (static chunks) + ceil(N/C)*C (A5, same closed form as the block-level model)
    cfg = it.Config(n_blocks=n, chunk=C, poll=1, k_steps=2, kpoll=1, worker_sm=ws, num_sms=2)
    r = it.explore(cfg)
    assert r.violations == set() and r.preempted_epoch_ends == 0
    st = it.initial_state(cfg)
    while True:                          # one trajectory to the end
        succ = it.successors(cfg, st)
        if not succ:
            break
        st = succ[0][1]
    assert st[9] == it.ST_DONE and st[6] == (1,) * n and st[5] == (2,) * n
    assert st[0] == len(ws) * C + -(-n // C) * C
