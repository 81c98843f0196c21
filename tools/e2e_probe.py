"""Where does the e2e time go? The bench's e2e protocol (managed HPF, relay CTA, host buffers
copied in before the victim starts, HP launched right after the victim's started hint), with the
victim's per-step device timeline: relay copy of the request, first / last yield exit, epoch end,
all mapped to the host clock through the started hint (the host thread waits in flep_sync, as the
bench does; the logs are read after the step, keep_logs). One JSON line per setting.

  python tools/e2e_probe.py [steps]
"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import bench as B
    from paper_conf_asplos_wulzj17_b200 import flep as F
    steps = int(sys.argv[1]) if len(sys.argv) > 1 else 30
    wl = B.Workload(torch)
    for spec in (1, 0, 1, 0):
        rt = F.Runtime(policy=F.POLICY_HPF, keep_logs=True)
        kLP = rt.register_kernel(F.BODY_SPMV_CSR_F32, chunk=1, poll=1, name="spmv", model=(0, 0, 0, 0, 70_000),
                                 started_hint=True, host_relay=True, spec_fetch=bool(spec))
        kHP = rt.register_kernel(F.BODY_STENCIL5_F32, chunk=1, poll=4, name="stencil", model=(0, 0, 0, 0, 30_000),
                                 clc=True)
        A = torch.cuda.Stream(priority=0)
        Bs = torch.cuda.Stream(priority=-2)
        lp_args = F.spmv_args(wl.d_y, wl.d_rowptr, wl.d_col, wl.d_val, wl.d_x)
        hp_args = F.stencil_args(wl.d_out, wl.d_in)
        rows = []
        for i in range(steps + 2):
            h_lp = rt.launch(kLP, F.spmv_grid(B.SPMV_ROWS), lp_args, priority=0, stream=A)
            t_w = time.perf_counter()
            while rt.query(h_lp).started_epoch < 1 and time.perf_counter() - t_w < 1.0:
                pass
            t_started_seen = F.now_ns()
            h_hp = rt.launch(kHP, F.stencil_grid(B.STENCIL_N), hp_args, priority=1, stream=Bs)
            rt.sync(h_hp, timeout_ns=10_000_000_000)
            rt.sync(h_lp, timeout_ns=10_000_000_000)
            info = rt.query(h_lp)
            if i < 2 or info.epoch < 2:
                continue
            ev = rt.events(h_lp, 1)
            ep = rt.epoch_info(h_lp, 1)
            w = [e for e in ev if e.t_entry > 0]
            off = t_started_seen - min(e.t_entry for e in w)
            ys = [e.t_exit for e in w if e.reason == F.REASON_YIELD]
            req = info.t_last_request
            rows.append({
                "e2e": (info.t_last_drain - req) / 1e3,
                "relay": (ep.relay_t_exit + off - req) / 1e3 if ep.relay_t_exit else None,
                "first_yield": (min(ys) + off - req) / 1e3 if ys else None,
                "last_yield": (max(ys) + off - req) / 1e3 if ys else None,
                "epoch_end": (ep.t_end + off - req) / 1e3,
                "seen": (info.t_last_drain - req) / 1e3,
                "yields": len(ys), "workers": len(w),
                "entry_spread": (max(e.t_entry for e in w) - min(e.t_entry for e in w)) / 1e3,
            })
        rt.close()
        med = {k: round(float(np.median([r[k] for r in rows if r[k] is not None])), 3)
               for k in rows[0] if rows and rows[0][k] is not None} if rows else {}
        print(json.dumps({"spec_fetch": spec, "steps": len(rows), "p50_us_after_request": med}), flush=True)


if __name__ == "__main__":
    main()
