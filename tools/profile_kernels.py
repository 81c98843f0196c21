"""Run each hot kernel (wrapped and unwrapped) a few times for ncu captures.

Usage under gpurun:  ncu --set full -k regex:flep_ ... python tools/profile_kernels.py [--kernels spmv,stencil]
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from synth import gen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--kernels", default="spmv,stencil,saxpy")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--chunk", type=int, default=1)
    ap.add_argument("--prefetch", type=int, default=1)
    ap.add_argument("--poll", type=int, default=1)
    ap.add_argument("--combos", default="", help="C:K:prefetch[:async[:clc[:spec]]][,...] wrapped variants (overrides --chunk/--poll/--prefetch)")
    a = ap.parse_args()
    import torch
    from paper_conf_asplos_wulzj17_b200 import build, flep as F
    build.build()
    rt = F.Runtime(exec_on_user_stream=True)
    sys.path.insert(0, ROOT)
    from bench import L2Flush
    flush = L2Flush(torch)
    T = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()  # noqa: E731
    jobs = []
    if "spmv" in a.kernels:
        rp, col, val, x = gen.csr_inputs(1 << 20, seed=2)
        y = torch.zeros(1 << 20, device="cuda")
        dev = (T(rp), T(col), T(val), T(x))        # kept alive: the args struct holds raw pointers
        args = F.spmv_args(y, *dev)
        jobs.append(("spmv", F.BODY_SPMV_CSR_F32, F.spmv_grid(1 << 20), args, dev + (y,)))
    if "stencil" in a.kernels:
        st = T(gen.stencil_f32_input(4096, seed=3))
        out = torch.empty_like(st)
        jobs.append(("stencil", F.BODY_STENCIL5_F32, F.stencil_grid(4096), F.stencil_args(out, st), (st, out)))
    if "saxpy" in a.kernels:
        n = 1 << 28
        xs = torch.ones(n, dtype=torch.int32, device="cuda")
        ys = torch.ones(n, dtype=torch.int32, device="cuda")
        jobs.append(("saxpy", F.BODY_SAXPY_I32, F.saxpy_grid(n), F.saxpy_i32_args(ys, xs, 3), (xs, ys)))
    if "gemm" in a.kernels:
        M = 8192
        A = (torch.rand(M, M, device="cuda") * 2 - 1).to(torch.bfloat16)
        B = (torch.rand(M, M, device="cuda") * 2 - 1).to(torch.bfloat16)
        Cg = torch.empty(M, M, device="cuda", dtype=torch.bfloat16)
        jobs.append(("gemm", F.BODY_GEMM_BF16, F.gemm_grid(M, M), F.gemm_args(Cg, A, B), (A, B, Cg)))
    s = torch.cuda.current_stream()
    combos = [(tuple(map(int, c.split(":"))) + (0, 0, 0))[:6] for c in a.combos.split(",")] if a.combos \
        else [(a.chunk, a.poll, a.prefetch, 0, 0, 0)]
    for name, body, grid, args, keep in jobs:
        ks = [rt.register_kernel(body, chunk=C, poll=K, prefetch=bool(pf), async_poll=bool(ap), clc=bool(clc),
                                 spec_fetch=bool(sp))
              for C, K, pf, ap, clc, sp in combos]
        for _ in range(a.reps):
            flush.zero_()
            rt.launch_unwrapped(body, grid, args, stream=s)
            torch.cuda.synchronize()
            for k in ks:
                flush.zero_()
                h = rt.launch(k, grid, args, stream=s)
                rt.sync(h)
    torch.cuda.synchronize()
    rt.close()


if __name__ == "__main__":
    main()
