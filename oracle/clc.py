"""Step model of the CLC task fetch (R25) and an exhaustive explorer.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

The launch is the original grid in chunks: CTA i stands for the original blocks [iC, iC+C). The
hardware keeps the CTAs that have not started in a queue; a free slot (one of W resident slots,
each on an SM) takes one of them, and a running CTA may cancel one with try_cancel instead and
run that chunk itself. The worker program (flep_device.cuh flep_clc_worker), in the order of its
steps:

  b = own chunk
  loop:
    every K chunks: poll the request word; if it names this SM (temporal n >= S, or
        rank[sm] < n, reading R6) -> stop
    if not stop: try_cancel -> claims one queued CTA's chunk c (or finds the queue empty)
    run chunk b                                 (every claimed chunk is run: reading A4)
    if a chunk c was claimed: b = c, continue; else leave

Which queued CTA the hardware launches or hands to a cancel is left open (any one), so the
explorer covers every order. Environment steps: a request (preempt n) and its withdrawal (resume)
at any point. There is no counter, no exit accounting and no relaunch: the launch is complete
when the queue is empty and every worker has left.

Properties (checked by tests/test_oracle_clc.py): every original block runs exactly once on every
interleaving, including runs where the request is never withdrawn (the queued CTAs still start,
one chunk each); a worker leaves with reason YIELD only if the request in force names its SM; a
planted bug that drops a claimed chunk on a stop is caught.
"""
from __future__ import annotations

from dataclasses import dataclass

FREE, START, CANCEL, RUN = range(4)
R_NONE, R_YIELD, R_EMPTY = 0, 1, 2


@dataclass(frozen=True)
class Config:
    n_blocks: int              # N original blocks
    chunk: int                 # C blocks per CTA of the CLC grid
    poll: int                  # K chunks between polls
    slot_sm: tuple             # SM of each resident slot (W = len)
    num_sms: int               # S
    preempt_widths: tuple = ()
    max_events: int = 0
    allow_resume: bool = True
    bug_drop_claimed_on_stop: bool = False

    @property
    def n_ctas(self):
        return -(-self.n_blocks // self.chunk)


def _names(cfg: Config, n: int, sm: int) -> bool:
    return n > 0 and (n >= cfg.num_sms or sm < n)


def initial_state(cfg: Config):
    # slot: (pc, b, claimed, k, stop, reason): b = chunk in hand, claimed = chunk taken by cancel
    # (or -1), k = chunks since the last poll, stop = the request word that stopped it (0: none)
    slots = tuple((FREE, -1, -1, 0, 0, R_NONE) for _ in cfg.slot_sm)
    # (queue of CTA ids not started, slots, cov, request n, events used, yield log)
    return (frozenset(range(cfg.n_ctas)), slots, (0,) * cfg.n_blocks, 0, 0, ())


def successors(cfg: Config, st):
    queue, slots, cov, req, ev, ylog = st
    out = []
    for i, (pc, b, claimed, k, stop, reason) in enumerate(slots):
        sm = cfg.slot_sm[i]

        def put(new, queue=queue, cov=cov, ylog=ylog, i=i):
            return (queue, slots[:i] + (new,) + slots[i + 1:], cov, req, ev, ylog)
        if pc == FREE:
            for c in sorted(queue):                       # the hardware starts a queued CTA here
                out.append((f"s{i}.launch{c}", put((START, c, -1, 0, 0, R_NONE), queue=queue - {c})))
        elif pc == START:                                  # the scheduling step before the body
            k2 = k + 1
            if k2 == cfg.poll:
                k2 = 0
                if _names(cfg, req, sm):
                    out.append((f"s{i}.poll_stop", put((RUN, b, -1, k2, req, R_YIELD))))
                    continue
            out.append((f"s{i}.poll", put((CANCEL, b, -1, k2, 0, R_NONE))))
        elif pc == CANCEL:                                 # try_cancel: any queued CTA, or none
            if queue:
                for c in sorted(queue):
                    out.append((f"s{i}.cancel{c}", put((RUN, b, c, k, 0, R_NONE), queue=queue - {c})))
            else:
                out.append((f"s{i}.cancel_empty", put((RUN, b, -1, k, 0, R_EMPTY))))
        elif pc == RUN:                                    # run the chunk in hand
            lo, hi = b * cfg.chunk, min(b * cfg.chunk + cfg.chunk, cfg.n_blocks)
            cov2 = list(cov)
            for x in range(lo, hi):
                cov2[x] += 1
            cov2 = tuple(cov2)
            drop = cfg.bug_drop_claimed_on_stop and claimed >= 0 and _names(cfg, req, sm)
            if claimed >= 0 and not drop:
                out.append((f"s{i}.run", put((START, claimed, -1, k, 0, R_NONE), cov=cov2)))
            else:
                why, seen = (R_YIELD, req) if drop else (reason, stop)
                out.append((f"s{i}.run_leave", put((FREE, -1, -1, 0, 0, R_NONE), cov=cov2,
                                                   ylog=ylog + ((sm, why, seen),))))
    if ev < cfg.max_events:
        for n in cfg.preempt_widths:
            if n != req:
                out.append((f"preempt({n})", (queue, slots, cov, n, ev + 1, ylog)))
        if cfg.allow_resume and req:
            out.append(("resume", (queue, slots, cov, 0, ev + 1, ylog)))
    return out


def check_state(cfg: Config, st) -> set:
    queue, slots, cov, req, ev, ylog = st
    v = set()
    if any(c > 1 for c in cov):
        v.add("block executed more than once")
    for sm, why, r in ylog:
        if why == R_YIELD and not _names(cfg, r, sm):
            v.add("I3: yield on an SM the request did not name")
    return v


@dataclass
class ExploreResult:
    states: int
    terminals: int
    violations: set
    yields_seen: int


def explore(cfg: Config, limit: int = 2_000_000) -> ExploreResult:
    """Every interleaving of slot steps, hardware choices and requests; checks the invariants on
    every state and, at every terminal state, that the launch completed with coverage == 1."""
    def canon(st):
        queue, slots, cov, req, ev, ylog = st
        return (queue, slots, cov, req, ev, tuple(sorted(set(ylog))))
    start = canon(initial_state(cfg))
    seen, stack = {start}, [start]
    violations, terminals, yields = set(), 0, 0
    while stack:
        st = stack.pop()
        violations |= check_state(cfg, st)
        succ = successors(cfg, st)
        if any(y[1] == R_YIELD for y in st[5]):
            yields += 1
        # a state where only request events remain is terminal for the launch
        if not [s for lab, s in succ if not lab.startswith(("preempt", "resume"))]:
            terminals += 1
            if st[0] or any(s[0] != FREE for s in st[1]) or any(c != 1 for c in st[2]):
                violations.add("liveness: launch ended with blocks not run exactly once")
        for _, s2 in succ:
            s2 = canon(s2)
            if s2 not in seen:
                if len(seen) >= limit:
                    raise RuntimeError("state limit exceeded")
                seen.add(s2)
                stack.append(s2)
    return ExploreResult(len(seen), terminals, violations, yields)
