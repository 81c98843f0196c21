"""Does a CLC persistent victim give up SMs to a higher-priority grid WITHOUT a FLEP request?

LP: SAXPY-i32 2^27 (~250 us) on a low-priority stream, as a CLC kernel or as the atomic-counter
worker; no preemption request is ever issued. HP: SAXPY-i32 2^20 launched on a high-priority
stream ~50 us after the LP starts (a spin kernel in front of it on its own stream). Prints, per
variant, the HP's start relative to its release (device %globaltimer of the spin's end is not
available, so: HP first CTA - LP first CTA) and whether the HP finished before the LP.
"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    from paper_conf_asplos_wulzj17_b200 import build, flep as F
    build.build()
    rt = F.Runtime(exec_on_user_stream=True)
    lo, hi = torch.cuda.Stream(priority=0), torch.cuda.Stream(priority=-2)
    n, n2 = 1 << 27, 1 << 20
    x = torch.randint(-2 ** 31, 2 ** 31 - 1, (n,), dtype=torch.int32, device="cuda")
    y = torch.zeros_like(x)
    x2 = torch.randint(-2 ** 31, 2 ** 31 - 1, (n2,), dtype=torch.int32, device="cuda")
    y2 = torch.zeros_like(x2)
    k_hp = rt.register_kernel(F.BODY_SAXPY_I32, chunk=4, poll=1)
    variants = {"clc": rt.register_kernel(F.BODY_SAXPY_I32, poll=4, clc=True),
                "counter": rt.register_kernel(F.BODY_SAXPY_I32, chunk=4, poll=1)}
    for name, k in variants.items():
        rows = []
        for rep in range(12):
            torch.cuda.synchronize()
            e0 = torch.cuda.Event()
            e0.record(lo)
            h = rt.launch(k, F.saxpy_grid(n), F.saxpy_i32_args(y, x, 3), stream=lo)
            hi.wait_event(e0)
            with torch.cuda.stream(hi):
                torch.cuda._sleep(100000)                # ~50 us
            h2 = rt.launch(k_hp, F.saxpy_grid(n2), F.saxpy_i32_args(y2, x2, 5), stream=hi)
            rt.sync(h2, timeout_ns=10_000_000_000)
            rt.sync(h, timeout_ns=10_000_000_000)
            torch.cuda.synchronize()
            lp, hp = rt.events(h, 1), rt.events(h2, 1)
            g = max(e.epoch for e in lp)
            lp = [e for e in lp if e.epoch == g]
            lp0, lp1 = min(e.t_entry for e in lp), max(e.t_exit for e in lp)
            hp0, hp1 = min(e.t_entry for e in hp), max(e.t_exit for e in hp)
            rows.append({"hp_start_after_lp_start_us": (hp0 - lp0) / 1e3, "hp_end_after_lp_start_us": (hp1 - lp0) / 1e3,
                         "lp_last_first_wave_exit_us": (lp1 - lp0) / 1e3,
                         "first_wave_yields": sum(1 for e in lp if e.reason == F.REASON_YIELD)})
        r = rows[2:]
        print(json.dumps({"variant": name,
                          "hp_start_after_lp_start_us_p50": float(np.median([a["hp_start_after_lp_start_us"] for a in r])),
                          "hp_end_after_lp_start_us_p50": float(np.median([a["hp_end_after_lp_start_us"] for a in r])),
                          "lp_first_wave_last_exit_us_p50": float(np.median([a["lp_last_first_wave_exit_us"] for a in r])),
                          "first_wave_yields": [a["first_wave_yields"] for a in r]}), flush=True)
    rt.close()


if __name__ == "__main__":
    main()
