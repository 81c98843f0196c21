"""Host-observed preemption latency breakdown (manual mode): flep_preempt() on a running wrapped
kernel -> host sees the PREEMPTED status. Also reports the device-side drain from the worker log."""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    from paper_conf_asplos_wulzj17_b200 import build, flep as F
    build.build()
    body = os.environ.get("BODY", "saxpy")
    flags = (F.FLAG_STREAM_MEMOP,) if body == "spmv" else (F.FLAG_STREAM_MEMOP, F.FLAG_HOST_MAPPED)
    for flag in flags:
        rt = F.Runtime(exec_on_user_stream=False, flag=flag)
        if body == "spmv":                       # the bench's victim: SpMV-CSR 2^22 rows, C = K = 1
            from synth import gen
            rows = 1 << 22
            rp, col, val, xv = gen.csr_inputs(rows, seed=2)
            T = lambda a: torch.from_numpy(a).cuda()  # noqa: E731
            yv = torch.zeros(rows, device="cuda")
            k = rt.register_kernel(F.BODY_SPMV_CSR_F32, chunk=1, poll=1, started_hint=True)
            keep = (T(rp), T(col), T(val), T(xv))   # outlive the args struct (raw pointers)
            grid, kargs = F.spmv_grid(rows), F.spmv_args(yv, *keep)
        else:
            n = 1 << 28
            x = torch.ones(n, dtype=torch.int32, device="cuda")
            y = torch.ones(n, dtype=torch.int32, device="cuda")
            k = rt.register_kernel(F.BODY_SAXPY_I32, chunk=8, poll=1, started_hint=True)
            grid, kargs = F.saxpy_grid(n), F.saxpy_i32_args(y, x, 1)
        lat, dev = [], []
        for r in range(30):
            h = rt.launch(k, grid, kargs)
            t0 = time.perf_counter()
            while rt.query(h).started_epoch < 1 and time.perf_counter() - t0 < 1:
                pass
            time.sleep(50e-6)
            t1 = F.now_ns()
            rt.preempt(h, rt.num_sms)
            while rt.query(h).state not in (F.STATE_PREEMPTED, F.STATE_DONE):
                pass
            t2 = F.now_ns()
            info = rt.query(h)
            if info.state == F.STATE_PREEMPTED:
                ev = rt.events(h, 1)
                ys = [e.t_exit for e in ev if e.reason == F.REASON_YIELD]
                if ys:
                    dev.append((max(ys) - min(ys)) / 1e3)
                lat.append((t2 - t1) / 1e3)
                rt.resume(h)
            rt.sync(h)
        print(json.dumps({"body": body, "flag": "stream_memop" if flag == F.FLAG_STREAM_MEMOP else "host_mapped",
                          "host_latency_us_p50": round(float(np.median(lat)), 2) if lat else None,
                          "min": round(min(lat), 2) if lat else None,
                          "yield_exit_spread_us_p50": round(float(np.median(dev)), 2) if dev else None,
                          "n": len(lat)}), flush=True)
        rt.close()


if __name__ == "__main__":
    main()
