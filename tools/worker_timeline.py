"""Per-worker timeline of one wrapped launch from the device event log (%globaltimer)."""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from synth import gen  # noqa: E402


COMBOS = [(tuple(map(int, c.split(":"))) + (0,))[:4] for c in
          (sys.argv[1] if len(sys.argv) > 1 else "1:1:0,2:1:1").split(",")]   # C:K:prefetch


def main():
    import torch
    from paper_conf_asplos_wulzj17_b200 import build, flep as F
    build.build()
    rt = F.Runtime(exec_on_user_stream=True, coverage=False)
    sys.path.insert(0, ROOT)
    from bench import L2Flush
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
    # device "stamps": a 1-block wrapped SAXPY before and after the target launch
    xs = torch.ones(256, dtype=torch.int32, device="cuda")
    ys = torch.ones(256, dtype=torch.int32, device="cuda")
    kst = rt.register_kernel(F.BODY_SAXPY_I32, chunk=1, poll=1)

    def stamp():
        hh = rt.launch(kst, (1, 1, 1), F.saxpy_i32_args(ys, xs, 1), stream=s)
        return hh

    for name, body, grid, args in cases:
        flush.zero_()
        h0 = stamp()
        rt.launch_unwrapped(body, grid, args, stream=s)
        h1 = stamp()
        rt.sync(h1)
        a = rt.events(h0, 1)[0]
        b = rt.events(h1, 1)[0]
        print(json.dumps({"body": name, "variant": "unwrapped", "stamp_gap_us": round((b.t_entry - a.t_exit) / 1e3, 2)}))
        for C, K, pf, ap in COMBOS:
            k = rt.register_kernel(body, chunk=C, poll=K, prefetch=bool(pf), async_poll=bool(ap))
            for rep in range(3):
                flush.zero_()
                h0 = stamp()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                h = rt.launch(k, grid, args, stream=s)
                e1.record(s)
                h1 = stamp()
                e1.synchronize()
                rt.sync(h1)
                ev = rt.events(h, 1)
                sa, sb = rt.events(h0, 1)[0], rt.events(h1, 1)[0]
                rt.sync(h)
            t0 = min(e.t_entry for e in ev)
            entry = np.array([e.t_entry - t0 for e in ev]) / 1e3
            exit_ = np.array([e.t_exit - t0 for e in ev]) / 1e3
            nb = np.array([e.n_blocks for e in ev])
            print(json.dumps({"body": name, "C": C, "K": K, "prefetch": pf, "async_poll": ap, "event_us": round(e0.elapsed_time(e1) * 1e3, 2),
                              "stamp_gap_us": round((sb.t_entry - sa.t_exit) / 1e3, 2),
                              "gap_before_us": round((t0 - sa.t_exit) / 1e3, 2),
                              "gap_after_us": round((sb.t_entry - max(e.t_exit for e in ev)) / 1e3, 2),
                              "workers": len(ev), "entry_max_us": round(entry.max(), 2),
                              "exit_min_us": round(exit_.min(), 2), "exit_p50_us": round(float(np.median(exit_)), 2),
                              "exit_max_us": round(exit_.max(), 2), "blocks_min": int(nb.min()), "blocks_max": int(nb.max()),
                              "blocks_mean": round(float(nb.mean()), 2)}), flush=True)
    rt.close()


if __name__ == "__main__":
    main()
