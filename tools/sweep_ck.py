"""(C, K, prefetch, CTAs/SM) sweep: wrapped vs unwrapped time per body, L2 flushed between reps.
The paper tunes its amortizing factor L offline as the smallest value keeping the overhead
under 4%; this is the B200 analogue over the chunk size C and poll period K."""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from synth import gen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--bodies", default="spmv,stencil,saxpy")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--chunks", default="1,2,4,8")
    ap.add_argument("--polls", default="1")
    ap.add_argument("--cps", default="0")
    ap.add_argument("--prefetch", default="0,1")
    ap.add_argument("--in-tile", default="0", help="GEMM: in-tile preemption variants (0,1)")
    ap.add_argument("--async-poll", default="0", help="async poll variants (0,1)")
    ap.add_argument("--warp", default="0", help="warp-task worker variants (0,1; R30)")
    ap.add_argument("--gate-us", type=float, default=0.0,
                    help="spin the stream this long before the start event (hides host submission latency)")
    a = ap.parse_args()
    import torch
    from paper_conf_asplos_wulzj17_b200 import build, flep as F
    build.build()
    rt = F.Runtime(exec_on_user_stream=True)
    sys.path.insert(0, ROOT)
    from bench import L2Flush
    flush = L2Flush(torch)
    T = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()  # noqa: E731
    jobs = {}
    if "spmv" in a.bodies.split(","):
        rp, col, val, x = gen.csr_inputs(1 << 20, seed=2)
        y = torch.zeros(1 << 20, device="cuda")
        dev = (T(rp), T(col), T(val), T(x))        # kept alive: the args struct holds raw pointers
        jobs["spmv"] = (F.BODY_SPMV_CSR_F32, F.spmv_grid(1 << 20), F.spmv_args(y, *dev),
                        8 * int(rp[-1]) + 12 * (1 << 20), dev + (y,))
    if "spmvvec" in a.bodies:
        rp, col, val, x = gen.csr_inputs(1 << 20, seed=2)
        y = torch.zeros(1 << 20, device="cuda")
        dev2 = (T(rp), T(col), T(val), T(x))
        jobs["spmvvec"] = (F.BODY_SPMV_CSR_F32_VEC, F.spmv_grid(1 << 20), F.spmv_args(y, *dev2),
                           8 * int(rp[-1]) + 12 * (1 << 20), dev2 + (y,))
    if "stencil" in a.bodies.split(","):
        st = T(gen.stencil_f32_input(4096, seed=3))
        out = torch.empty_like(st)
        jobs["stencil"] = (F.BODY_STENCIL5_F32, F.stencil_grid(4096), F.stencil_args(out, st), 8 * 4096 * 4096, (st, out))
    if "stencil16k" in a.bodies:
        st = torch.rand(16384, 16384, device="cuda")
        out = torch.empty_like(st)
        jobs["stencil16k"] = (F.BODY_STENCIL5_F32, F.stencil_grid(16384), F.stencil_args(out, st), 8 * 16384 ** 2, (st, out))
    if "gemm" in a.bodies:
        M = 8192
        A = torch.randn(M, M, device="cuda").to(torch.bfloat16)
        B = torch.randn(M, M, device="cuda").to(torch.bfloat16)
        Cg = torch.empty(M, M, device="cuda", dtype=torch.bfloat16)
        jobs["gemm"] = (F.BODY_GEMM_BF16, F.gemm_grid(M, M), F.gemm_args(Cg, A, B), 2 * M ** 3, (A, B, Cg))
        for _ in range(3):
            torch.matmul(A, B.t())
        ts = []
        for _ in range(10):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            torch.matmul(A, B.t())
            e1.record()
            e1.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e3)
        print(json.dumps({"body": "gemm", "variant": "cublas(torch.matmul)", "us": round(float(np.median(ts)), 3),
                          "tflops": round(2 * M ** 3 / float(np.median(ts)) / 1e6, 1)}), flush=True)
    if "saxpy" in a.bodies:
        n = 1 << 28
        xs = torch.ones(n, dtype=torch.int32, device="cuda")
        ys = torch.ones(n, dtype=torch.int32, device="cuda")
        jobs["saxpy"] = (F.BODY_SAXPY_I32, F.saxpy_grid(n), F.saxpy_i32_args(ys, xs, 3), 12 * n, (xs, ys))
    s = torch.cuda.current_stream()

    def timed(fn):
        ts = []
        for r in range(a.reps + 2):
            flush.zero_()
            if a.gate_us > 0:
                torch.cuda._sleep(int(a.gate_us * 2000))
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            h = fn()
            e1.record(s)
            e1.synchronize()
            if h is not None:
                rt.sync(h)
            if r >= 2:
                ts.append(e0.elapsed_time(e1) * 1e3)
        return float(np.median(ts))

    for name, (body, grid, args, nbytes, keep) in jobs.items():
        tu = timed(lambda: rt.launch_unwrapped(body, grid, args, stream=s))
        print(json.dumps({"body": name, "variant": "unwrapped", "us": round(tu, 3),
                          ("tflops" if name == "gemm" else "gbs"): round(nbytes / tu / (1e6 if name == "gemm" else 1e3), 1)}), flush=True)
        for C in map(int, a.chunks.split(",")):
            for K in map(int, a.polls.split(",")):
                for pf in map(int, a.prefetch.split(",")):
                    for cps in map(int, a.cps.split(",")):
                      for it_ in (map(int, a.in_tile.split(",")) if name == "gemm" else [0]):
                       for ap_ in map(int, a.async_poll.split(",")):
                        for wp in map(int, a.warp.split(",")):
                         if it_ and pf:
                            continue
                         if wp and body not in (F.BODY_SPMV_CSR_F32_VEC, F.BODY_STENCIL5_F32):
                            continue
                         k = rt.register_kernel(body, chunk=C, poll=K, prefetch=bool(pf), ctas_per_sm=cps,
                                               in_tile=bool(it_), async_poll=bool(ap_), warp_tasks=bool(wp))
                         tw = timed(lambda: rt.launch(k, grid, args, stream=s))
                         print(json.dumps({"body": name, "C": C, "K": K, "prefetch": pf, "cps": cps, "in_tile": it_,
                                          "async_poll": ap_, "warp": wp,
                                          "us": round(tw, 3),
                                          ("tflops" if name == "gemm" else "gbs"): round(nbytes / tw / (1e6 if name == "gemm" else 1e3), 1),
                                          "overhead_pct": round((tw / tu - 1) * 100, 2)}), flush=True)
    rt.close()


if __name__ == "__main__":
    main()
