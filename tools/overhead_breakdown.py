"""Where does a short wrapped kernel lose time against its unwrapped twin? For each (C, K, prefetch,
async) variant of the 4096^2 stencil (configs[1] HP) and the SpMV (configs[1] LP): CUDA-event
duration (L2 flushed), and from the device worker log (%globaltimer): first entry -> last entry
(grid ramp), first entry -> last exit (device span), first exit -> last exit (tail), per-worker
blocks (min / max). Prints one JSON line per case.

  python tools/overhead_breakdown.py [C:K:pf:ap,...]
"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from synth import gen  # noqa: E402


def main():
    import torch
    from paper_conf_asplos_wulzj17_b200 import build, flep as F
    from paper_conf_asplos_wulzj17_b200.calibrate import dither, event_mean_us
    from bench import L2Flush
    build.build()
    # C:K:prefetch:async[:sched_warp]
    combos = [(tuple(map(int, c.split(":"))) + (0,))[:5] for c in
              (sys.argv[1] if len(sys.argv) > 1 else "1:1:0:0,2:1:1:1,4:1:0:0,8:1:0:0").split(",")]
    rt = F.Runtime(exec_on_user_stream=True)
    flush = L2Flush(torch)
    T = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()  # noqa: E731
    st = T(gen.stencil_f32_input(4096, seed=3))
    out = torch.empty_like(st)
    rp, col, val, x = gen.csr_inputs(1 << 20, seed=2)
    dev = (T(rp), T(col), T(val), T(x))   # outlive the args structs (raw pointers)
    y = torch.zeros(1 << 20, device="cuda")
    cases = [("stencil", F.BODY_STENCIL5_F32, F.stencil_grid(4096), F.stencil_args(out, st)),
             ("spmv", F.BODY_SPMV_CSR_F32, F.spmv_grid(1 << 20), F.spmv_args(y, *dev))]
    s = torch.cuda.current_stream()
    reps = 30

    def timed(fn):
        ts, hs = [], []
        for r in range(reps + 2):
            flush.zero_()
            dither(torch, int(os.environ.get("DITHER_BASE", "0")))
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            h = fn()
            e1.record(s)
            e1.synchronize()
            if h is not None:
                rt.sync(h)
            if r >= 2:
                ts.append(e0.elapsed_time(e1) * 1e3)
                hs.append(h)
        return ts, hs

    for name, body, grid, args in cases:
        tu, _ = timed(lambda: rt.launch_unwrapped(body, grid, args, stream=s))
        print(json.dumps({"body": name, "variant": "unwrapped", "event_us": round(event_mean_us(tu), 3),
                          "event_min_us": round(min(tu), 3)}), flush=True)
        for C, K, pf, ap, sw in combos:
            kk = rt.register_kernel(body, chunk=C, poll=K, prefetch=bool(pf), async_poll=bool(ap), sched_warp=bool(sw))
            tw, hs = timed(lambda: rt.launch(kk, grid, args, stream=s))
            ev = rt.events(hs[-1], 1)
            ent = np.array([e.t_entry for e in ev], dtype=np.int64)
            ext = np.array([e.t_exit for e in ev], dtype=np.int64)
            nb = np.array([e.n_blocks for e in ev])
            t0 = ent.min()
            print(json.dumps({
                "body": name, "variant": "wrapped", "C": C, "K": K, "prefetch": pf, "async_poll": ap, "sched_warp": sw,
                "workers": len(ev), "event_us": round(event_mean_us(tw), 3), "event_min_us": round(min(tw), 3),
                "ramp_us": round((ent.max() - t0) / 1e3, 3),
                "span_us": round((ext.max() - t0) / 1e3, 3),
                "tail_us": round((ext.max() - ext.min()) / 1e3, 3),
                "exit_p10_us": round((np.percentile(ext, 10) - t0) / 1e3, 3),
                "blocks_min": int(nb.min()), "blocks_max": int(nb.max())}), flush=True)
    rt.close()


if __name__ == "__main__":
    main()
