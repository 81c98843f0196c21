"""A/B of wrapper-overhead experiments: runs the configs[1] kernels (SpMV CSR-stream and CSR-vector,
stencil5 4096^2) wrapped and unwrapped, interleaved and dithered, L2 flushed, with the library given
by FLEP_LIB_PATH (a prebuilt variant), and reports per case the CUDA-event mean and the device span
of the workers (first entry -> last exit, %globaltimer) so that launch / teardown time outside the
span is visible.

  FLEP_LIB_PATH=build_variants/x.so python tools/ab_overhead.py [case,...]
case = body:C:K[:pf[:clc[:warp[:in_chunk[:static[:async_poll[:spec_fetch]]]]]]]   (static = 1: the static
       persistent twin U1 with chunk C instead of the FLEP worker)
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
    from paper_conf_asplos_wulzj17_b200 import flep as F
    from paper_conf_asplos_wulzj17_b200.calibrate import dither, event_mean_us
    from bench import L2Flush
    cases = (sys.argv[1] if len(sys.argv) > 1 else
             "spmv:1:1,spmv:2:1,spmvvec:1:1,spmvvec:2:1,stencil:1:1,stencil:1:4:0:1").split(",")
    tag = os.path.basename(os.environ.get("FLEP_LIB_PATH", "libflep.so"))
    rt = F.Runtime(exec_on_user_stream=True)
    flush = L2Flush(torch)
    T = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()  # noqa: E731
    keep = []
    rp, col, val, x = gen.csr_inputs(1 << 20, seed=2)
    dev = [T(rp), T(col), T(val), T(x)]
    y = torch.zeros(1 << 20, device="cuda")
    keep += dev + [y]
    st = T(gen.stencil_f32_input(4096, seed=3))
    out = torch.empty_like(st)
    keep += [st, out]
    bodies = {"spmv": (F.BODY_SPMV_CSR_F32, F.spmv_grid(1 << 20), F.spmv_args(y, *dev)),
              "spmvvec": (F.BODY_SPMV_CSR_F32_VEC, F.spmv_grid(1 << 20), F.spmv_args(y, *dev)),
              "stencil": (F.BODY_STENCIL5_F32, F.stencil_grid(4096), F.stencil_args(out, st))}
    s = torch.cuda.current_stream()
    utrace = torch.zeros(2 * 70000, dtype=torch.int64, device="cuda")
    try:
        rt.set_trace(None, utrace)                 # FLEP_TRACE builds: per-block entry/exit of unwrapped grids
        traced = True
    except F.FlepError:
        traced = False
    reps = int(os.environ.get("AB_REPS", "40"))
    gate = int(float(os.environ.get("AB_GATE_US", "0")) * 1965)    # SM cycles at the max clock
    for c in cases:
        f = c.split(":")
        name, C, K = f[0], int(f[1]), int(f[2])
        pf, clc, warp = (int(f[3]) if len(f) > 3 else 0), (int(f[4]) if len(f) > 4 else 0), (int(f[5]) if len(f) > 5 else 0)
        ic = int(f[6]) if len(f) > 6 else 0
        u1 = int(f[7]) if len(f) > 7 else 0
        ap = int(f[8]) if len(f) > 8 else 0
        sp = int(f[9]) if len(f) > 9 else 0
        body, grid, args = bodies[name]
        k = rt.register_kernel(body, chunk=C, poll=K, prefetch=bool(pf), clc=bool(clc), warp_tasks=bool(warp),
                               in_chunk=bool(ic), async_poll=bool(ap), spec_fetch=bool(sp))
        tw, tu, span, uspan = [], [], [], []
        for r in range(reps + 3):
            for mode in ("w", "u"):
                flush.zero_()
                dither(torch)
                if gate:
                    torch.cuda._sleep(gate)      # GPU busy while the host submits e0 + the kernel
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                if mode == "w" and u1:
                    rt.launch_static(body, grid, args, chunk=C, stream=s)
                    h = None
                elif mode == "w":
                    h = rt.launch(k, grid, args, stream=s)
                else:
                    rt.launch_unwrapped(body, grid, args, stream=s)
                e1.record(s)
                e1.synchronize()
                if mode == "w" and h is not None:
                    rt.sync(h)
                if r >= 3:
                    (tw if mode == "w" else tu).append(e0.elapsed_time(e1) * 1e3)
                    if mode == "u" and traced:
                        nb = grid[0] * grid[1]
                        tr = utrace[:2 * nb].view(nb, 2)
                        uspan.append(float((tr[:, 1].max() - tr[:, 0].min()).item()) / 1e3)
                    if mode == "w" and not clc and h is not None:
                        ev = [e for e in rt.events(h, 1) if e.t_entry > 0]
                        if ev:
                            a0, a1 = min(e.t_entry for e in ev), max(e.t_exit for e in ev)
                            span.append((a1 - a0) / 1e3)
        w, u = event_mean_us(tw), event_mean_us(tu)
        print(json.dumps({"lib": tag, "gate_us": float(os.environ.get("AB_GATE_US", "0")), "case": c, "wrapped_us": round(w, 3), "unwrapped_us": round(u, 3),
                          "overhead_pct": round((w / u - 1) * 100, 2),
                          "worker_span_us": round(float(np.median(span)), 3) if span else None,
                          "outside_span_us": round(w - float(np.median(span)), 3) if span else None,
                          "unwrapped_span_us": round(float(np.median(uspan)), 3) if uspan else None,
                          "unwrapped_outside_span_us": round(u - float(np.median(uspan)), 3) if uspan else None}), flush=True)
    rt.close()


if __name__ == "__main__":
    main()
