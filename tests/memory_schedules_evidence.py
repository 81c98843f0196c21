"""Evidence run (GPU): many random manual preempt/resume schedules on the configs[1] bodies as the
bench runs them (speculative fetch, R34): the SpMV victim (2^20 rows) and the 5-point stencil
(4096^2, fp32) at the configs[1] sizes, each schedule checked for exactly-once coverage, I3 on every epoch and an output
bit-identical to the uninterrupted run. Test infrastructure (uses tests/flep_gpu_util.py); one
JSON line. Usage: python tests/memory_schedules_evidence.py [schedules per body]"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from flep_gpu_util import flep_mod, run_manual_schedule, t  # noqa: E402
from synth import gen  # noqa: E402


def main():
    import torch
    n_sched = int(sys.argv[1]) if len(sys.argv) > 1 else 1000
    f = flep_mod()
    rt = f.Runtime(coverage=True)
    rows = 1 << 20
    rp, col, val, x = gen.csr_inputs(rows, seed=61)
    keep = (t(rp), t(col), t(val), t(x))
    ys = torch.zeros(rows, device="cuda")
    st_in = t(gen.stencil_f32_input(4096, seed=62))
    st_out = torch.zeros_like(st_in)
    cases = (("spmv_spec_fetch", f.BODY_SPMV_CSR_F32, f.spmv_grid(rows), f.spmv_args(ys, *keep), ys),
             ("stencil_f32_spec_fetch", f.BODY_STENCIL5_F32, f.stencil_grid(4096), f.stencil_args(st_out, st_in), st_out))
    out = {"what": f"{n_sched} random manual schedules per body (gen.preempt_schedule: 1-4 cycles, temporal or "
                   "spatial widths, C in {1, 2} and K random), speculative fetch", "bodies": {}}
    for name, body, grid, args, o in cases:
        nb = grid[0] * grid[1]
        rt.launch_unwrapped(body, grid, args)
        torch.cuda.synchronize()
        ref = o.clone()
        kern, bad, pre = {}, [], 0
        for i in range(n_sched):
            s = gen.preempt_schedule(15000 + i, nb, rt.num_sms)
            key = (min(s["C"], 2), s["K"])
            if key not in kern:
                kern[key] = rt.register_kernel(body, chunk=key[0], poll=key[1], spec_fetch=True)
            o.zero_()
            h, npre, viol = run_manual_schedule(rt, kern[key], grid, args, nb, s, rt.num_sms, check_prefix=False)
            pre += npre
            if not np.all(rt.coverage_np(h, nb) == 1):
                viol.append("I1: coverage != 1")
            torch.cuda.synchronize()
            if not torch.equal(o, ref):
                viol.append("output differs from the uninterrupted run")
            if viol:
                bad.append({"i": i, "schedule": s, "violations": viol[:3]})
        out["bodies"][name] = {"schedules": n_sched, "blocks": nb, "violations": len(bad), "preempted_epochs": pre,
                               "first_bad": bad[:2]}
    rt.close()
    print(json.dumps(out))


if __name__ == "__main__":
    main()
