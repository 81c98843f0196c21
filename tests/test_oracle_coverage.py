"""Pins for oracle/coverage.py: exhaustive interleavings on tiny instances
(Fig. 2's 2 SMs x 2 CTAs), hand-traced trajectories, a closed form for the final counter,
temporal-equivalence of n >= num_sms, and a planted bug the checker must catch."""
import itertools

import pytest

from oracle import coverage as cv


def _cfg(**kw):
    base = dict(n_blocks=5, chunk=1, poll=1, worker_sm=(0, 0, 1, 1), num_sms=2,
                preempt_widths=(1, 2), max_events=2)
    base.update(kw)
    return cv.Config(**base)


@pytest.mark.parametrize("C,K", list(itertools.product([1, 2], [1, 2])))
def test_exhaustive_no_violations_fig2(C, K):
    # Fig. 2: two SMs, two CTAs each; up to 2 preempt events (spatial 1 SM or temporal)
    r = cv.explore(_cfg(n_blocks=5 if (C, K) != (1, 2) else 4, chunk=C, poll=K))
    assert r.violations == set()
    assert r.terminals > 0
    assert r.preempted_epoch_ends > 0      # preempted epochs really are explored


@pytest.mark.parametrize("C,K", [(1, 1), (1, 2), (2, 1)])
def test_exhaustive_prefetch_no_violations(C, K):
    # chunk prefetch (R3): a stopping worker still runs the chunk it holds
    r = cv.explore(_cfg(n_blocks=4 if C == 1 else 5, chunk=C, poll=K, worker_sm=(0, 0, 1), prefetch=True))
    assert r.violations == set()
    assert r.preempted_epoch_ends > 0


def test_prefetch_final_counter_closed_form():
    for n, C, ws in [(5, 1, (0, 0, 1, 1)), (7, 2, (0, 1))]:
        r = cv.explore(cv.Config(n_blocks=n, chunk=C, poll=1, worker_sm=ws, num_sms=2, prefetch=True))
        assert r.violations == set()
        assert r.terminal_ctrs == {cv.final_counter_no_preempt(n, C, len(ws))}


@pytest.mark.parametrize("C", [1, 2])
def test_exhaustive_spatial_refill(C):
    # flep_refill: widen a spatial request to temporal and queue a full-width epoch; when the
    # running epoch completes the launch first (and the device cleans the block), the queued
    # epoch must exit without fetching (completed-generation marker)
    r = cv.explore(_cfg(n_blocks=4 if C == 1 else 5, chunk=C, poll=1, worker_sm=(0, 0, 1),
                        preempt_widths=(1,), max_events=2, allow_refill=True))
    assert r.violations == set()


def test_refill_without_done_marker_double_executes():
    # the same exploration with the marker check disabled finds double executions: the check is
    # what keeps a refill that races the last blocks exactly-once
    import oracle.coverage as m
    orig = m.successors

    def no_marker(cfg, st):
        st2 = st[:9] + ((st[9][0], 0, st[9][2]) + st[9][3:],)   # pretend no epoch ever recorded completion
        return [(lab, s[:9] + ((s[9][0], 0, s[9][2]) + s[9][3:],)) for lab, s in orig(cfg, st2)]
    m.successors = no_marker
    try:
        r = cv.explore(_cfg(n_blocks=3, chunk=1, poll=1, worker_sm=(0, 1), preempt_widths=(1,),
                            max_events=2, allow_refill=True))
    finally:
        m.successors = orig
    assert any("more than once" in v for v in r.violations)


def test_exhaustive_with_clear_events():
    r = cv.explore(_cfg(n_blocks=6, chunk=2, poll=2, allow_clear=True))
    assert r.violations == set()


def test_planted_bug_is_caught():
    r = cv.explore(_cfg(bug_exit_holding_chunk=True))
    assert any(v.startswith("I1") for v in r.violations)
    assert any(v.startswith("I2") for v in r.violations)


def test_final_counter_closed_form_without_preemption():
    for n, C, ws in [(5, 1, (0, 0, 1, 1)), (5, 2, (0, 1)), (7, 3, (0, 0, 1)), (4, 4, (0,))]:
        r = cv.explore(cv.Config(n_blocks=n, chunk=C, poll=1, worker_sm=ws, num_sms=2))
        assert r.violations == set()
        assert r.terminal_ctrs == {cv.final_counter_no_preempt(n, C, len(ws))}


def test_temporal_equivalence_n_ge_num_sms():
    # I4 / P:174: spa_P >= number of SMs behaves exactly as temporal preemption
    a = cv.explore(_cfg(preempt_widths=(2,), max_events=1))
    b = cv.explore(_cfg(preempt_widths=(7,), max_events=1))
    assert (a.states, a.terminals, a.terminal_ctrs, a.preempted_epoch_ends) == \
           (b.states, b.terminals, b.terminal_ctrs, b.preempted_epoch_ends)


def _pick(seq):
    """Choose successors by label prefix in order; falls back to the first successor."""
    it = iter(seq)
    want = [next(it, None)]

    def choose(labels):
        w = want[0]
        if w is not None:
            for i, lab in enumerate(labels):
                if lab == w:
                    want[0] = next(it, None)
                    return i
        return 0
    return choose


def test_hand_traced_temporal_preempt_after_one_chunk():
    # one worker on SM0, N=3, C=1, K=1: poll, fetch b0, process, preempt, poll -> yield.
    cfg = cv.Config(n_blocks=3, chunk=1, poll=1, worker_sm=(0,), num_sms=2,
                    preempt_widths=(2,), max_events=1)
    st = cv.initial_state(cfg)
    for lab in ["w0.poll", "w0.fetch", "w0.proc", "preempt(2)", "w0.poll", "w0.exit"]:
        st = dict(cv.successors(cfg, st))[lab]
    ctr, ctrl, done, exited, cov, epoch, status, workers, ev, extra = st
    assert status == cv.ST_PREEMPTED and cov == (1, 0, 0) and ctr == 1 and done == 1
    assert list(cov) == cv.expected_prefix(ctr, 3)
    # resume: a fresh epoch ignores the stale request (gen 0) and finishes the rest
    st = dict(cv.successors(cfg, st))["resume"]
    for lab in ["w0.poll", "w0.fetch", "w0.proc", "w0.poll", "w0.fetch", "w0.proc", "w0.poll",
                "w0.fetch", "w0.exit"]:
        st = dict(cv.successors(cfg, st))[lab]
    assert st[6] == cv.ST_DONE and st[4] == (1, 1, 1) and st[9][2] == 4 and st[0] == 0


def test_hand_traced_spatial_keeps_other_sm_running():
    # workers on SM0 and SM1, spatial request n=1 yields SM0 only (rank = smid)
    cfg = cv.Config(n_blocks=4, chunk=1, poll=1, worker_sm=(0, 1), num_sms=2,
                    preempt_widths=(1,), max_events=1)
    st = cv.initial_state(cfg)
    for lab in ["preempt(1)", "w0.poll", "w1.poll", "w0.exit"]:
        st = dict(cv.successors(cfg, st))[lab]
    workers = st[7]
    assert workers[0][3] == cv.R_YIELD and workers[1][0] == cv.FETCH
    for lab in ["w1.fetch", "w1.proc", "w1.poll", "w1.fetch", "w1.proc", "w1.poll", "w1.fetch",
                "w1.proc", "w1.poll", "w1.fetch", "w1.proc", "w1.poll", "w1.fetch", "w1.exit"]:
        st = dict(cv.successors(cfg, st))[lab]
    assert st[6] == cv.ST_DONE and st[4] == (1, 1, 1, 1)
    assert st[7][1][3] == cv.R_EXHAUSTED


def test_expected_prefix():
    assert cv.expected_prefix(0, 3) == [0, 0, 0]
    assert cv.expected_prefix(2, 3) == [1, 1, 0]
    assert cv.expected_prefix(9, 3) == [1, 1, 1]


# ---- static first chunks (R20): the product wrapper's first epoch -------------------

@pytest.mark.parametrize("C,K,pf", [(1, 1, False), (1, 2, False), (2, 1, False), (1, 1, True), (2, 1, True)])
def test_exhaustive_static_first_no_violations(C, K, pf):
    ws = (0, 1) if pf else (0, 0, 1)
    # enough blocks that a request can still find work after the static chunks (and the first
    # K-chunk period, and a prefetched chunk)
    r = cv.explore(_cfg(n_blocks=len(ws) * C * (K + pf) + 1, chunk=C, poll=K, worker_sm=ws,
                        prefetch=pf, static_first=True))
    assert r.violations == set()
    assert r.preempted_epoch_ends > 0


@pytest.mark.parametrize("n,C,ws", [(5, 1, (0, 0, 1, 1)), (7, 2, (0, 1)), (2, 1, (0, 0, 1, 1)),
                                    (3, 2, (0, 0, 1)), (4, 4, (0,))])
def test_static_first_final_counter_closed_form(n, C, ws):
    # every worker holding a static chunk below N runs it and then fails exactly one fetch;
    # workers whose static chunk starts at or beyond N leave at once: the effective counter is
    # W*C + ceil(N/C)*C, the same closed form as with dynamic first fetches (A5)
    for pf in (False, True):
        r = cv.explore(cv.Config(n_blocks=n, chunk=C, poll=1, worker_sm=ws, num_sms=2, prefetch=pf,
                                 static_first=True))
        assert r.violations == set()
        assert r.terminal_ctrs == {cv.final_counter_no_preempt(n, C, len(ws))}


def test_static_first_spatial_refill():
    r = cv.explore(_cfg(n_blocks=7, chunk=1, poll=1, worker_sm=(0, 0, 1), preempt_widths=(1,),
                        max_events=2, allow_refill=True, static_first=True))
    assert r.violations == set()


def test_hand_traced_static_first_preempt():
    # two workers, N=5, C=1: both run their static chunks (blocks 0 and 1) without polling; a
    # temporal request then stops both at their first poll. The drained epoch covers [0, 2) and
    # the counter (W*C = 2) names exactly that prefix; the resume finishes blocks 2..4.
    cfg = cv.Config(n_blocks=5, chunk=1, poll=1, worker_sm=(0, 1), num_sms=2, preempt_widths=(2,),
                    max_events=1, static_first=True)
    st = cv.initial_state(cfg)
    assert st[0] == 2
    for lab in ["w0.fetch", "w1.fetch", "preempt(2)", "w0.proc", "w1.proc", "w0.poll", "w1.poll",
                "w0.exit", "w1.exit"]:
        st = dict(cv.successors(cfg, st))[lab]
    ctr, ctrl, done, exited, cov, epoch, status, workers, ev, extra = st
    assert status == cv.ST_PREEMPTED and cov == (1, 1, 0, 0, 0) and ctr == 2 and done == 2
    st = dict(cv.successors(cfg, st))["resume"]
    assert st[7][0][0] == cv.POLL and st[7][0][4] == cv.NOCHUNK     # later epochs poll first
    while True:
        succ = cv.successors(cfg, st)
        if not succ:
            break
        st = succ[0][1]
    assert st[6] == cv.ST_DONE and st[4] == (1, 1, 1, 1, 1)


# ---- async poll (R22): the poll tests the word copied when the previous chunk was taken

@pytest.mark.parametrize("C,K,pf,sf", [(1, 1, False, False), (2, 1, False, True), (1, 2, False, True),
                                       (1, 1, True, True), (2, 1, True, False)])
def test_exhaustive_async_poll_no_violations(C, K, pf, sf):
    ws = (0, 1) if pf else (0, 0, 1)
    n = len(ws) * C * (K + pf) + 1 if sf else 4 + C
    r = cv.explore(_cfg(n_blocks=n, chunk=C, poll=K, worker_sm=ws, prefetch=pf, static_first=sf,
                        async_poll=True))
    assert r.violations == set()
    assert r.preempted_epoch_ends > 0


def test_async_poll_refill_and_clear():
    r = cv.explore(_cfg(n_blocks=5, chunk=1, poll=1, worker_sm=(0, 0, 1), preempt_widths=(1,),
                        max_events=2, allow_refill=True, static_first=True, async_poll=True))
    assert r.violations == set()
    r = cv.explore(_cfg(n_blocks=6, chunk=2, poll=2, allow_clear=True, async_poll=True))
    assert r.violations == set()


def test_hand_traced_async_poll_acts_one_chunk_later():
    # one worker, N=4, C=K=1: the request lands after the worker took block 0, so the copy taken
    # with block 0 misses it: the worker still fetches block 1 and leaves at the poll after it
    # (a synchronous poll would have left before block 1)
    cfg = cv.Config(n_blocks=4, chunk=1, poll=1, worker_sm=(0,), num_sms=2, preempt_widths=(2,),
                    max_events=1, async_poll=True)
    st = cv.initial_state(cfg)
    for lab in ["w0.poll", "w0.fetch", "preempt(2)", "w0.proc", "w0.poll", "w0.fetch", "w0.proc",
                "w0.poll", "w0.exit"]:
        st = dict(cv.successors(cfg, st))[lab]
    assert st[6] == cv.ST_PREEMPTED and st[4] == (1, 1, 0, 0) and st[0] == 2
    sync = cv.Config(n_blocks=4, chunk=1, poll=1, worker_sm=(0,), num_sms=2, preempt_widths=(2,),
                     max_events=1)
    st = cv.initial_state(sync)
    for lab in ["w0.poll", "w0.fetch", "preempt(2)", "w0.proc", "w0.poll", "w0.exit"]:
        st = dict(cv.successors(sync, st))[lab]
    assert st[6] == cv.ST_PREEMPTED and st[4] == (1, 0, 0, 0)


# ---- exit accounting by the exhausted fetch (R23) -----------------------------------

def _early_done_states(cfg):
    """Reachable states where DONE is published while some worker still runs a held chunk."""
    start = cv._canon(cfg, cv.initial_state(cfg))
    seen, stack, early = {start}, [start], 0
    while stack:
        st = stack.pop()
        if st[6] == cv.ST_DONE and not cv._all_gone(st[7]) and any(w[0] == cv.PROC for w in st[7]):
            early += 1
        for _, s2 in cv.successors(cfg, st):
            s2 = cv._canon(cfg, s2)
            if s2 not in seen:
                seen.add(s2)
                stack.append(s2)
    return early


def test_done_published_early_is_reached_and_safe():
    # with prefetch the W-th exit event can be an exhausted prefetch: DONE is then published
    # while its issuer (and others) still run their last chunks; I6 holds in every such state
    cfg = _cfg(n_blocks=5, chunk=1, poll=1, worker_sm=(0, 1), prefetch=True, static_first=True)
    assert _early_done_states(cfg) > 0
    assert cv.explore(cfg).violations == set()


def test_first_exhausted_value_formula():
    # the device formula: multiples of C from the epoch start (W*C with static first chunks)
    cfg = cv.Config(n_blocks=7, chunk=2, poll=1, worker_sm=(0, 1), num_sms=2, static_first=True)
    assert cv._first_exhausted(cfg, 0) == 8 and cv._first_exhausted(cfg, 1) == 8
    cfg = cv.Config(n_blocks=3, chunk=2, poll=1, worker_sm=(0, 0, 1), num_sms=2, static_first=True)
    assert cv._first_exhausted(cfg, 0) == 6 and cv._first_exhausted(cfg, 1) == 4


def test_planted_double_count_is_caught():
    # counting a worker's exit twice lets an early event look like the W-th: the epoch is
    # published while a worker can still fetch (or never published at all)
    for pf in (False, True):
        cfg = _cfg(n_blocks=5, chunk=1, poll=1, worker_sm=(0, 0, 1), prefetch=pf, bug_count_twice=True)
        assert cv.explore(cfg).violations


# ---- speculative fetch (R34): fetch + poll together, a fetched chunk returned -----------

@pytest.mark.parametrize("n,c,k,sms,extra", [
    (4, 1, 1, (0, 1), {}), (5, 2, 1, (0, 1), {}), (6, 1, 1, (0, 1, 1), {}),
    (6, 1, 1, (0, 1, 1), {"allow_clear": True}), (6, 1, 1, (0, 1, 1), {"allow_refill": True}),
    (5, 1, 2, (0, 0, 1), {}),
])
def test_spec_fetch_exhaustive(n, c, k, sms, extra):
    cfg = cv.Config(n_blocks=n, chunk=c, poll=k, worker_sm=sms, num_sms=2, preempt_widths=(1, 2),
                    max_events=3, static_first=True, spec_fetch=True, **extra)
    r = cv.explore(cfg)
    assert r.violations == set()
    assert r.preempted_epoch_ends > 0


@pytest.mark.parametrize("bug", ["bug_spec_drop", "bug_spec_publish"])
def test_spec_fetch_planted_bugs_caught(bug):
    cfg = cv.Config(n_blocks=4, chunk=1, poll=1, worker_sm=(0, 1), num_sms=2, preempt_widths=(1, 2),
                    max_events=2, static_first=True, spec_fetch=True, **{bug: True})
    r = cv.explore(cfg)
    assert any(v.startswith("I1") for v in r.violations)


def test_spec_fetch_hand_trace():
    """N = 4, C = 1, two workers on SMs 0 and 1 (R20 static first chunks 0 and 1, counter at 2).
    w0 runs block 0, fetches block 2 speculatively, a temporal request lands, w0's poll sees it:
    block 2 goes to w0's record and w0 leaves; w1 (holding its static block 1) runs it, then its
    poll step sees the request and leaves. The drained epoch covered {0, 1}: the prefix [0, 3)
    minus the record. On resume, worker 0 runs block 2 from its record first (after its entry
    check), then both fetch; every block once."""
    cfg = cv.Config(n_blocks=4, chunk=1, poll=1, worker_sm=(0, 1), num_sms=2, preempt_widths=(2,),
                    max_events=1, static_first=True, spec_fetch=True)
    st = cv.initial_state(cfg)
    for lab in ["w0.fetch", "w0.proc", "w0.spec_fetch", "preempt(2)", "w0.spec_yield", "w0.exit",
                "w1.fetch", "w1.proc", "w1.spec_fetch", "w1.spec_yield", "w1.exit"]:
        st = dict(cv.successors(cfg, st))[lab]
    assert st[6] == cv.ST_PREEMPTED
    assert st[4] == (1, 1, 0, 0)
    assert st[9][3] == (2, 3)                          # both fetched chunks were returned
    assert st[0] == 4                                  # counter: 2 static + 2 speculative fetches
    assert cv.check_state(cfg, st) == set()
    st = dict(cv.successors(cfg, st))["resume"]
    for lab in ["w0.take_rest", "w0.proc", "w1.take_rest", "w1.proc"]:
        st = dict(cv.successors(cfg, st))[lab]
    assert st[4] == (1, 1, 1, 1) and st[9][3] == (cv.NOCHUNK, cv.NOCHUNK)
    while True:                                        # the rest: exhausted fetches and exits
        succ = cv.successors(cfg, st)
        if not succ:
            break
        st = succ[0][1]
    assert st[6] == cv.ST_DONE and st[4] == (1, 1, 1, 1)
