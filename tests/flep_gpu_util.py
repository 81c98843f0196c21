"""Shared helpers for the GPU tests: build the library, make tensors from the seeded generators,
run manual preempt/resume schedules, check the wrapper invariants."""
from __future__ import annotations

import numpy as np

from oracle import coverage as cov_oracle
from synth import gen

_built = False


def flep_mod():
    global _built
    from paper_conf_asplos_wulzj17_b200 import build, flep
    if not _built:
        build.build()
        _built = True
    return flep


def t(a, dev="cuda"):
    import torch
    return torch.from_numpy(np.ascontiguousarray(a)).to(dev)


def saxpy_i32_case(n, seed):
    x, y = gen.saxpy_i32_inputs(n, seed)
    return x, y


def run_manual_schedule(rt, kernel, grid, args, n_blocks, schedule, num_sms, check_prefix=True,
                        priority=0, stats=None):
    """Execute one manual-mode preempt/resume schedule driven by device self-triggers.

    schedule = dict(cycles=[(t_star, n_sms), ...]). Returns (handle, n_preempted_epochs,
    violations list). The caller checks outputs and final coverage."""
    f = flep_mod()
    cycles = list(schedule["cycles"])
    violations = []
    if cycles:
        t0, n0 = cycles.pop(0)
        rt.arm_next_trigger(t0, n0)
        cur_n = n0
    else:
        cur_n = 0
    h = rt.launch(kernel, grid, args, priority=priority)
    preempted = 0
    while True:
        rt.wait_epoch(h, timeout_ns=20_000_000_000)
        info = rt.query(h)
        epoch = info.epoch
        ev = rt.events(h, epoch)
        for e in ev:
            if e.reason == f.REASON_YIELD:
                if not (cur_n >= num_sms or e.smid < cur_n):
                    violations.append(f"I3: worker on SM {e.smid} yielded under n={cur_n}")
            elif e.reason != f.REASON_EXHAUSTED:
                violations.append(f"bad exit reason {e.reason}")
        if info.state == f.STATE_DONE:
            break
        if info.state != f.STATE_PREEMPTED:
            violations.append(f"unexpected state {info.state}")
            break
        preempted += 1
        if stats is not None and info.blocks_done < min(int(info.counter), n_blocks):
            stats["partial_epochs"] = stats.get("partial_epochs", 0) + 1   # fetched but unfinished
        if check_prefix:
            c = rt.coverage_np(h, n_blocks)
            exp = np.array(cov_oracle.expected_prefix(int(info.counter), n_blocks), dtype=np.uint32)
            if not np.array_equal(c, exp):
                violations.append(f"I2: coverage after preempted epoch {epoch} is not the prefix of ctr={info.counter}")
        if cycles:
            tn, nn = cycles.pop(0)
            rt.trigger_at(h, tn, nn)
            cur_n = nn
        else:
            cur_n = 0
        rt.resume(h)
    rt.sync(h, timeout_ns=20_000_000_000)
    return h, preempted, violations
