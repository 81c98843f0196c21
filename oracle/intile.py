"""Step model of in-tile preemption (R21) and an exhaustive explorer.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

The paper preempts at block (task) granularity: a pulled task is always processed (Fig. 4,
P:132-162; A4). For a long contraction block the B200 wrapper also lets a worker stop INSIDE a
block between two k-steps of its accumulation: the partial accumulator is saved with the k-step
reached, and the worker with the same index in the next epoch restores it and continues. This
module models that protocol at k-step granularity, independently of the CUDA code:

  worker w, epoch e (first epoch: static first chunk [w*C, w*C+C), R20):
    if e > 0 and rec[w].valid:                    # a stopped block from the previous epoch
        if poll() names my SM: exit (the record stays for a later epoch)
        take rec[w] (valid = 0): continue block rec.b at k-step rec.kb, then blocks
        rec.b+1 .. rec.b_end-1 of its chunk
    loop: poll every K chunks (Fig. 4(b)); fetch a chunk (pull_task);
          for each block b of the chunk: for each k-step kb:
              every KP k-steps (not at the first): in-tile poll; if it names my SM:
                  rec[w] = (1, b, kb, chunk end); exit
              accumulate k-step kb of b
          block done: write b's result once (epilogue), done += 1

Shared state: ctr (effective counter), ctrl = (gen, n), done, exited, claim[b] (chunk handed
out: coverage log), acc[b] (k-steps accumulated), wr[b] (results written), rec[w].
Invariants checked on every reachable state:
  J1 k-steps of a block accumulate in order and exactly once (acc[b] only ever moves by +1
     from the value the worker expects; checked in the step itself) and a block is written only
     when all K_STEPS are accumulated, at most once; at DONE every block written once;
  J2 a drained (PREEMPTED) epoch has claimed exactly the prefix [0, min(ctr, N));
  J3 yields only on requested SMs; J4 done == number of written blocks;
  liveness: every terminal state is DONE.
"""
from __future__ import annotations

from dataclasses import dataclass

# worker pcs
START, POLL, FETCH, KSTEP, EXIT, GONE = range(6)
R_NONE, R_YIELD, R_EXH = 0, 1, 2
ST_RUNNING, ST_PREEMPTED, ST_DONE, ST_LOST = 0, 1, 2, 3


@dataclass(frozen=True)
class Config:
    n_blocks: int
    chunk: int                    # C
    poll: int                     # K (chunks between block-boundary polls)
    k_steps: int                  # k-steps per block
    kpoll: int                    # KP: k-steps between in-tile polls
    worker_sm: tuple
    num_sms: int
    preempt_widths: tuple = ()
    max_events: int = 0
    min_left: int = 0             # do not stop when fewer than this many k-steps remain
    bug_restore_from_zero: bool = False     # planted: restore ignores rec.kb
    bug_drop_chunk_rest: bool = False       # planted: record b_end = b + 1 (rest of chunk lost)

    @property
    def W(self):
        return len(self.worker_sm)


def _stop(cfg, ctrl, epoch, sm):
    gen, n = ctrl
    if gen != epoch or n == 0:
        return False
    return n >= cfg.num_sms or sm < n


def _fresh_workers(cfg, first):
    # worker = (pc, i, b, kb, kb0, b_end, reason, restoring)
    #   i: chunks since the last block-boundary poll; b: block in progress; kb: next k-step;
    #   kb0: first k-step of this run of the block (in-tile polls count from it, as on the
    #   device); b_end: end of the chunk in progress
    if first:   # static first chunk (R20): no poll, no fetch
        out = []
        for w in range(cfg.W):
            s = w * cfg.chunk
            if s >= cfg.n_blocks:
                out.append((EXIT, 0, 0, 0, 0, 0, R_EXH, False))
            else:
                out.append((KSTEP, 1 % cfg.poll, s, 0, 0, min(s + cfg.chunk, cfg.n_blocks), R_NONE, False))
        return tuple(out)
    return tuple((START, 0, 0, 0, 0, 0, R_NONE, False) for _ in range(cfg.W))


def initial_state(cfg: Config):
    n = cfg.n_blocks
    ctr0 = cfg.W * cfg.chunk
    claim = tuple(1 if b < min(ctr0, n) else 0 for b in range(n))   # static chunks are handed out
    recs = tuple((0, 0, 0, 0) for _ in range(cfg.W))
    # (ctr, ctrl, done, exited, claim, acc, wr, recs, epoch, status, workers, events, bad)
    return (ctr0, (0, 0), 0, 0, claim, (0,) * n, (0,) * n, recs, 0, ST_RUNNING,
            _fresh_workers(cfg, True), 0, ())


def successors(cfg: Config, st):
    ctr, ctrl, done, exited, claim, acc, wr, recs, epoch, status, workers, ev, bad = st
    out = []
    n = cfg.n_blocks
    if status == ST_RUNNING:
        for w, wk in enumerate(workers):
            pc, i, b, kb, kb0, b_end, reason, restoring = wk
            sm = cfg.worker_sm[w]

            def put(nw, **kw):
                d = dict(ctr=ctr, done=done, exited=exited, claim=claim, acc=acc, wr=wr, recs=recs,
                         status=status, epoch=epoch, workers=None, bad=bad)
                d.update(kw)
                nws = d["workers"] if d["workers"] is not None else workers[:w] + (nw,) + workers[w + 1:]
                return (d["ctr"], ctrl, d["done"], d["exited"], d["claim"], d["acc"], d["wr"], d["recs"],
                        d["epoch"], d["status"], nws, ev, d["bad"])

            if pc == START:                       # later epochs: a record to continue?
                valid, rb, rkb, rend = recs[w]
                if valid:
                    if _stop(cfg, ctrl, epoch, sm):
                        out.append((f"w{w}.entry_yield", put((EXIT, 0, 0, 0, 0, 0, R_YIELD, False))))
                    else:
                        k0 = 0 if cfg.bug_restore_from_zero else rkb
                        r2 = recs[:w] + ((0, 0, 0, 0),) + recs[w + 1:]
                        out.append((f"w{w}.restore", put((KSTEP, 0, rb, k0, k0, rend, R_NONE, True), recs=r2)))
                else:
                    out.append((f"w{w}.start", put((POLL, 0, 0, 0, 0, 0, R_NONE, False))))
            elif pc == POLL:
                if i == 0 and _stop(cfg, ctrl, epoch, sm):
                    out.append((f"w{w}.poll", put((EXIT, 0, 0, 0, 0, 0, R_YIELD, False))))
                else:
                    out.append((f"w{w}.poll", put((FETCH, i, 0, 0, 0, 0, R_NONE, False))))
            elif pc == FETCH:
                s = ctr
                if s >= n:
                    out.append((f"w{w}.fetch", put((EXIT, 0, 0, 0, 0, 0, R_EXH, False), ctr=ctr + cfg.chunk)))
                else:
                    e = min(s + cfg.chunk, n)
                    cl = list(claim)
                    for bb in range(s, e):
                        cl[bb] += 1
                    i2 = (i + 1) % cfg.poll
                    out.append((f"w{w}.fetch", put((KSTEP, i2, s, 0, 0, e, R_NONE, False),
                                                   ctr=ctr + cfg.chunk, claim=tuple(cl))))
            elif pc == KSTEP:
                # in-tile poll before k-step kb: every KP k-steps of this run of the block, never
                # at its first k-step, and not when at most min_left k-steps remain
                j = kb - kb0
                if (j > 0 and j % cfg.kpoll == 0 and cfg.k_steps - kb > cfg.min_left
                        and _stop(cfg, ctrl, epoch, sm)):
                    end = b + 1 if cfg.bug_drop_chunk_rest else b_end
                    r2 = recs[:w] + ((1, b, kb, end),) + recs[w + 1:]
                    out.append((f"w{w}.intile_yield", put((EXIT, 0, 0, 0, 0, 0, R_YIELD, False), recs=r2)))
                # accumulate k-step kb of block b (J1: in order, exactly once)
                a = list(acc)
                bad2 = bad
                if a[b] != kb:
                    bad2 = bad + (f"J1: block {b} k-step {kb} accumulated with acc={a[b]}",)
                a[b] += 1
                if kb + 1 < cfg.k_steps:
                    out.append((f"w{w}.kstep", put((KSTEP, i, b, kb + 1, kb0, b_end, R_NONE, restoring),
                                                   acc=tuple(a), bad=bad2)))
                else:                              # block complete: epilogue writes once
                    wv = list(wr)
                    wv[b] += 1
                    if a[b] != cfg.k_steps:
                        bad2 = bad2 + (f"J1: block {b} written with {a[b]} k-steps",)
                    if b + 1 < b_end:
                        nw = (KSTEP, i, b + 1, 0, 0, b_end, R_NONE, restoring)
                    else:
                        nw = (POLL, i, 0, 0, 0, 0, R_NONE, False)
                    out.append((f"w{w}.kstep", put(nw, acc=tuple(a), wr=tuple(wv), done=done + 1, bad=bad2)))
            elif pc == EXIT:
                ex2 = exited + 1
                nw = (GONE, 0, 0, 0, 0, 0, reason, False)
                if ex2 == cfg.W:
                    if done == n:
                        st2 = ST_DONE
                    elif ctr < n or any(r[0] for r in recs):
                        st2 = ST_PREEMPTED
                    else:
                        st2 = ST_LOST
                    out.append((f"w{w}.exit", put(nw, exited=ex2, status=st2)))
                else:
                    out.append((f"w{w}.exit", put(nw, exited=ex2)))
        if ev < cfg.max_events:
            for nn in cfg.preempt_widths:
                if ctrl[0] != epoch or nn > ctrl[1]:
                    out.append((f"preempt({nn})", (ctr, (epoch, nn), done, exited, claim, acc, wr, recs, epoch,
                                                   status, workers, ev + 1, bad)))
    elif status == ST_PREEMPTED:
        out.append(("resume", (ctr, ctrl, done, 0, claim, acc, wr, recs, epoch + 1, ST_RUNNING,
                               _fresh_workers(cfg, False), ev, bad)))
    return out


def check_state(cfg: Config, st) -> set:
    ctr, ctrl, done, exited, claim, acc, wr, recs, epoch, status, workers, ev, bad = st
    v = set(bad)
    n = cfg.n_blocks
    if any(x > 1 for x in wr):
        v.add("J1: a block result written more than once")
    if any(x > cfg.k_steps for x in acc):
        v.add("J1: more k-steps than the block has")
    if status == ST_DONE and (any(x != 1 for x in wr) or any(x != cfg.k_steps for x in acc)):
        v.add("J1: DONE without every block written once")
    if any(c > 1 for c in claim):
        v.add("J2: a block handed out twice")
    if status == ST_PREEMPTED:
        m = min(ctr, n)
        if list(claim) != [1] * m + [0] * (n - m):
            v.add("J2: drained epoch did not claim a counter prefix")
    if status == ST_LOST:
        v.add("liveness: counter exhausted with blocks neither written nor recorded")
    if done != sum(wr):
        v.add("J4: done != blocks written")
    for w, wk in enumerate(workers):
        if wk[6] == R_YIELD and not _stop(cfg, ctrl, epoch, cfg.worker_sm[w]):
            v.add("J3: yield on a non-requested SM")
    return v


@dataclass
class ExploreResult:
    states: int
    terminals: int
    violations: set
    preempted_epoch_ends: int
    intile_yields: int


def explore(cfg: Config, limit: int = 3_000_000) -> ExploreResult:
    """Exhaustive DFS over all interleavings of worker steps and preempt/resume events."""
    start = initial_state(cfg)
    seen = {start}
    stack = [start]
    violations = set()
    terminals = 0
    pre = 0
    intile = 0
    while stack:
        st = stack.pop()
        violations |= check_state(cfg, st)
        if st[9] == ST_PREEMPTED:
            pre += 1
        succ = successors(cfg, st)
        if not succ:
            terminals += 1
            if st[9] != ST_DONE:
                violations.add("liveness: terminal state is not DONE")
            continue
        for lab, s2 in succ:
            if "intile_yield" in lab:
                intile += 1
            if s2 not in seen:
                if len(seen) >= limit:
                    raise RuntimeError("state limit exceeded")
                seen.add(s2)
                stack.append(s2)
    return ExploreResult(len(seen), terminals, violations, pre, intile)
