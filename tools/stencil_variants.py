"""Stencil5 fp32 bodies side by side (register path vs TMA-staged): unwrapped grid, counter worker
and CLC worker at 4096^2 (configs[1]) and 16384^2 (configs[2]); dithered CUDA-event means with the
L2 flushed before every launch. One JSON line per (n, body, variant) with GB/s of the 8 B/cell
algorithmic traffic."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    from paper_conf_asplos_wulzj17_b200 import build, flep as F
    from paper_conf_asplos_wulzj17_b200.calibrate import dither, event_mean_us
    from bench import L2Flush
    build.build()
    rt = F.Runtime(exec_on_user_stream=True)
    flush = L2Flush(torch)
    s = torch.cuda.current_stream()
    reps = int(os.environ.get("REPS", "30"))

    def timed(fn):
        ts = []
        for r in range(reps + 2):
            flush.zero_()
            dither(torch)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            h = fn()
            e1.record(s)
            e1.synchronize()
            if h is not None:
                rt.sync(h)
            if r >= 2:
                ts.append(e0.elapsed_time(e1) * 1e3)
        return event_mean_us(ts)
    for n in (4096, 16384):
        a = torch.rand(n, n, device="cuda")
        o = torch.empty_like(a)
        args, grid = F.stencil_args(o, a), F.stencil_grid(n)
        for bname, body in (("register", F.BODY_STENCIL5_F32), ("tma", F.BODY_STENCIL5_F32_TMA)):
            variants = [("unwrapped", None)]
            variants += [(f"counter_C{c}", dict(chunk=c, poll=1)) for c in (1, 2, 4)]
            variants += [("clc_C1_K4", dict(chunk=1, poll=4, clc=True)), ("clc_C2_K2", dict(chunk=2, poll=2, clc=True))]
            for vname, kw in variants:
                if kw is None:
                    us = timed(lambda: rt.launch_unwrapped(body, grid, args, stream=s))
                else:
                    k = rt.register_kernel(body, **kw)
                    us = timed(lambda: rt.launch(k, grid, args, stream=s))
                print(json.dumps({"n": n, "body": bname, "variant": vname, "us": round(us, 3),
                                  "gbs": round(8 * n * n / (us * 1e-6) / 1e9, 1)}), flush=True)
    rt.close()


if __name__ == "__main__":
    main()
