"""Where does the wrapper's time go? Per-chunk scheduling timestamps of the worker grids vs
per-block entry/exit of the unwrapped grids (diagnostics build, -DFLEP_TRACE; L2 flushed before
every launch). Prints one JSON line per (body, variant).

  unwrapped : block duration (entry -> exit of all threads), kernel span, slot utilisation
  wrapped   : per chunk, sched = tid 0's scheduling step (poll + fetch round trips), body = from
              the step's return to the next step (tid 0's share of the body + waiting at the
              chunk barrier for the slowest warp), span, and the tail (first worker exit -> last)
"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from synth import gen  # noqa: E402

KT = 64
KW = 5      # words per chunk record (flep_device.cuh kTraceWords)


def main():
    os.environ["FLEP_NVCC_EXTRA"] = (os.environ.get("FLEP_NVCC_EXTRA", "") + " -DFLEP_TRACE").strip()
    import torch
    from paper_conf_asplos_wulzj17_b200 import build, flep as F
    build.build(force=True)
    rt = F.Runtime(exec_on_user_stream=True)
    from bench import L2Flush
    flush = L2Flush(torch)
    T = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()  # noqa: E731
    st = T(gen.stencil_f32_input(4096, seed=3))
    out = torch.empty_like(st)
    rp, col, val, x = gen.csr_inputs(1 << 20, seed=2)
    y = torch.zeros(1 << 20, device="cuda")
    dev = [T(rp), T(col), T(val), T(x)]         # kept alive: the args structs hold raw pointers
    cases = [("stencil", F.BODY_STENCIL5_F32, F.stencil_grid(4096), F.stencil_args(out, st)),
             ("spmv", F.BODY_SPMV_CSR_F32, F.spmv_grid(1 << 20), F.spmv_args(y, *dev)),
             ("spmvvec", F.BODY_SPMV_CSR_F32_VEC, F.spmv_grid(1 << 20), F.spmv_args(y, *dev))]
    only = os.environ.get("TRACE_BODIES")
    if only:
        cases = [c for c in cases if c[0] in only.split(",")]
    s = torch.cuda.current_stream()
    combos = [(tuple(map(int, c.split(":"))) + (0,))[:4] for c in (sys.argv[1] if len(sys.argv) > 1 else "1:1:0,1:1:1").split(",")]
    for name, body, grid, args in cases:
        nb = grid[0] * grid[1] * grid[2]
        ut = torch.zeros(nb * 2, dtype=torch.int64, device="cuda")
        rt.set_trace(None, ut)
        res = []
        for rep in range(4):
            flush.zero_()
            torch.cuda.synchronize()
            rt.launch_unwrapped(body, grid, args, stream=s)
            torch.cuda.synchronize()
            u = ut.view(nb, 2).cpu().numpy().astype(np.int64)
            dur = (u[:, 1] - u[:, 0]) / 1e3
            span = (u[:, 1].max() - u[:, 0].min()) / 1e3
            res.append((span, float(np.mean(dur)), float(np.median(dur))))
        span, mdur, pdur = res[-1]
        k, w = rt.workers_for(body)
        print(json.dumps({"body": name, "variant": "unwrapped", "span_us": round(span, 2),
                          "block_us_mean": round(mdur, 3), "block_us_p50": round(pdur, 3),
                          "slot_utilisation": round(nb * mdur / (span * w), 3), "slots": w}), flush=True)
        rt.set_trace(None, None)
        for C, K, pf, ap in combos:
            kk = rt.register_kernel(body, chunk=C, poll=K, prefetch=bool(pf), async_poll=bool(ap))
            wt = torch.zeros(w * KT * KW, dtype=torch.int64, device="cuda")
            rt.set_trace(wt, None)
            for rep in range(4):
                wt.zero_()
                flush.zero_()
                torch.cuda.synchronize()
                h = rt.launch(kk, grid, args, stream=s)
                rt.sync(h, timeout_ns=5_000_000_000)
                torch.cuda.synchronize()
            rt.set_trace(None, None)
            tr = wt.view(w, KT, KW).cpu().numpy().astype(np.int64)
            ev = rt.events(h, 1)
            entry = np.array([e.t_entry for e in ev])
            exit_ = np.array([e.t_exit for e in ev])
            t0 = entry.min()
            sched, bodyt, first, pollt, fetcht, bart, issuet = [], [], [], [], [], [], []
            for i in range(w):
                ta, tp, tb, tc, tq = tr[i, :, 0], tr[i, :, 1], tr[i, :, 2], tr[i, :, 3], tr[i, :, 4]
                n = int(np.count_nonzero(ta))
                if n == 0:
                    continue
                sched.extend((tb[:n] - ta[:n]) / 1e3)
                pollt.extend((tp[:n] - ta[:n]) / 1e3)
                fetcht.extend((tq[:n] - tp[:n]) / 1e3)
                issuet.extend((tb[:n] - tq[:n]) / 1e3)
                bart.extend((tc[:n] - tb[:n]) / 1e3)
                bodyt.extend((ta[1:n] - tc[:n - 1]) / 1e3)
                first.append((tc[0] - t0) / 1e3)
            m = lambda v: round(float(np.mean(v)), 3) if len(v) else None  # noqa: E731
            print(json.dumps({"body": name, "variant": "wrapped", "C": C, "K": K, "prefetch": pf, "async_poll": ap,
                              "span_us": round((exit_.max() - t0) / 1e3, 2),
                              "sched_us_mean": m(sched),
                              "sched_us_p50": round(float(np.median(sched)), 3),
                              "poll_us_mean": m(pollt), "fetch_us_mean": m(fetcht), "issue_us_mean": m(issuet),
                              "barrier_wait_us_mean": m(bart),
                              "body_us_mean": m(bodyt),
                              "body_us_p50": round(float(np.median(bodyt)), 3),
                              "first_chunk_ready_us_p50": round(float(np.median(first)), 3),
                              "exit_first_us": round((exit_.min() - t0) / 1e3, 2),
                              "exit_last_us": round((exit_.max() - t0) / 1e3, 2),
                              "steps": len(sched)}), flush=True)
    rt.close()
    os.environ.pop("FLEP_NVCC_EXTRA", None)
    build.build(force=True)          # leave the normal library behind


if __name__ == "__main__":
    main()
