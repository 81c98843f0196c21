"""Evidence run (GPU): many random manual preempt/resume schedules on the tensor-core bodies with
in-tile preemption — the 1-CTA GEMM (R21), the 256x256 CTA pair (R32) and the 256x512 pair
(R35) — each schedule checked for exactly-once coverage of every tile, I3 on every epoch and a C
bit-identical to the uninterrupted run. Test infrastructure (uses tests/flep_gpu_util.py);
prints one JSON line. Usage: python tests/gemm_schedules_evidence.py [schedules per body]"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from flep_gpu_util import flep_mod, run_manual_schedule  # noqa: E402
from synth import gen  # noqa: E402


def main():
    import torch
    n_sched = int(sys.argv[1]) if len(sys.argv) > 1 else 300
    f = flep_mod()
    rt = f.Runtime(coverage=True)
    m, n, k = 2048, 4096, 2048
    a_bits, b_bits = gen.gemm_bf16_inputs(m, n, k, seed=990)
    A = torch.from_numpy(a_bits.view(np.int16)).cuda().view(torch.bfloat16)
    B = torch.from_numpy(b_bits.view(np.int16)).cuda().view(torch.bfloat16)
    out = {"what": f"{n_sched} random manual schedules per body (gen.preempt_schedule: 1-4 cycles, temporal or "
                   f"spatial widths, C and K random), GEMM {m}x{n}x{k} bf16, in-tile preemption",
           "bodies": {}}
    for name, body, grid_fn in (("gemm_1cta", f.BODY_GEMM_BF16, f.gemm_grid),
                                ("gemm_pair_256x256", f.BODY_GEMM_BF16_2SM, f.gemm2_grid),
                                ("gemm_pair_256x512", f.BODY_GEMM_BF16_2SM_W, f.gemm2w_grid)):
        grid = grid_fn(m, n)
        ntiles = grid[0] * grid[1]
        C0 = torch.empty((m, n), dtype=torch.bfloat16, device="cuda")
        rt.launch_unwrapped(body, grid, f.gemm_args(C0, A, B))
        torch.cuda.synchronize()
        C1 = torch.empty_like(C0)
        kern, bad, pre, stats = {}, [], 0, {}
        for i in range(n_sched):
            s = gen.preempt_schedule(12000 + i, ntiles, rt.num_sms)
            key = (min(s["C"], 2), s["K"])
            if key not in kern:
                kern[key] = rt.register_kernel(body, chunk=key[0], poll=key[1], in_tile=True)
            C1.fill_(float("nan"))
            h, npre, viol = run_manual_schedule(rt, kern[key], grid, f.gemm_args(C1, A, B), ntiles, s, rt.num_sms,
                                                check_prefix=False, stats=stats)
            pre += npre
            if not np.all(rt.coverage_np(h, ntiles) == 1):
                viol.append("I1: coverage != 1")
            if not torch.equal(C0.view(torch.int16), C1.view(torch.int16)):
                viol.append("C differs from the uninterrupted run")
            if viol:
                bad.append({"i": i, "schedule": s, "violations": viol[:3]})
        out["bodies"][name] = {"schedules": n_sched, "tiles": ntiles, "violations": len(bad),
                               "preempted_epochs": pre, "epochs_stopped_inside_a_tile": stats.get("partial_epochs", 0),
                               "first_bad": bad[:2]}
    rt.close()
    print(json.dumps(out))


if __name__ == "__main__":
    main()
