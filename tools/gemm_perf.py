"""GEMM 8192^3 (configs[3]'s largest): cuBLAS (torch.matmul) vs the 1-CTA body (unwrapped,
static persistent U1, FLEP worker) vs the CTA-pair body (unwrapped, U1, FLEP worker), interleaved
round-robin, CUDA events, clocks sampled during the run. One JSON line per variant."""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    from paper_conf_asplos_wulzj17_b200 import build, flep as F
    from bench import ClockSampler
    build.build()
    M = int(os.environ.get("GEMM_M", "8192"))
    reps = int(os.environ.get("GEMM_REPS", "12"))
    g = torch.Generator(device="cuda")
    g.manual_seed(5)
    A = (torch.rand(M, M, device="cuda", generator=g) * 2 - 1).to(torch.bfloat16)
    B = (torch.rand(M, M, device="cuda", generator=g) * 2 - 1).to(torch.bfloat16)
    C = torch.empty(M, M, device="cuda", dtype=torch.bfloat16)
    rt = F.Runtime(exec_on_user_stream=True)
    s = torch.cuda.current_stream()
    args = F.gemm_args(C, A, B)
    g1, g2, g2w = F.gemm_grid(M, M), F.gemm2_grid(M, M), F.gemm2w_grid(M, M)
    k1 = {c: rt.register_kernel(F.BODY_GEMM_BF16, chunk=c, poll=1) for c in (1, 2)}
    k1t = rt.register_kernel(F.BODY_GEMM_BF16, chunk=2, poll=1, in_tile=True)
    k2 = {c: rt.register_kernel(F.BODY_GEMM_BF16_2SM, chunk=c, poll=1) for c in (1, 2)}
    k2t = rt.register_kernel(F.BODY_GEMM_BF16_2SM, chunk=1, poll=1, in_tile=True)
    kw = {c: rt.register_kernel(F.BODY_GEMM_BF16_2SM_W, chunk=c, poll=1) for c in (1, 2)}
    kwt = rt.register_kernel(F.BODY_GEMM_BF16_2SM_W, chunk=1, poll=1, in_tile=True)
    variants = {
        "cublas": lambda: (torch.matmul(A, B.t(), out=C), None)[1],
        "gemm1_unwrapped": lambda: rt.launch_unwrapped(F.BODY_GEMM_BF16, g1, args, stream=s),
        "gemm1_static_u1": lambda: rt.launch_static(F.BODY_GEMM_BF16, g1, args, chunk=1, stream=s),
        "gemm1_flep_c1": lambda: rt.launch(k1[1], g1, args, stream=s),
        "gemm1_flep_c2": lambda: rt.launch(k1[2], g1, args, stream=s),
        "gemm1_flep_c2_intile": lambda: rt.launch(k1t, g1, args, stream=s),
        "gemm2_unwrapped": lambda: rt.launch_unwrapped(F.BODY_GEMM_BF16_2SM, g2, args, stream=s),
        "gemm2_static_u1": lambda: rt.launch_static(F.BODY_GEMM_BF16_2SM, g2, args, stream=s),
        "gemm2_flep_c1": lambda: rt.launch(k2[1], g2, args, stream=s),
        "gemm2_flep_c2": lambda: rt.launch(k2[2], g2, args, stream=s),
        "gemm2_flep_c1_intile": lambda: rt.launch(k2t, g2, args, stream=s),
        "gemm2w_unwrapped": lambda: rt.launch_unwrapped(F.BODY_GEMM_BF16_2SM_W, g2w, args, stream=s),
        "gemm2w_static_u1": lambda: rt.launch_static(F.BODY_GEMM_BF16_2SM_W, g2w, args, stream=s),
        "gemm2w_flep_c1": lambda: rt.launch(kw[1], g2w, args, stream=s),
        "gemm2w_flep_c2": lambda: rt.launch(kw[2], g2w, args, stream=s),
        "gemm2w_flep_c1_intile": lambda: rt.launch(kwt, g2w, args, stream=s),
    }
    only = os.environ.get("GEMM_ONLY")                 # comma list: a subset of the variants
    if only:
        variants = {k: v for k, v in variants.items() if k in only.split(",") or k == "cublas"}
    sustained = float(os.environ.get("GEMM_SUSTAINED_S", "0"))
    if sustained > 0:
        return run_sustained(torch, rt, variants, s, M, sustained)
    ts = {k: [] for k in variants}
    with ClockSampler(0) as clk:
        for r in range(reps + 2):
            for name, fn in variants.items():
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                h = fn()
                e1.record(s)
                e1.synchronize()
                if isinstance(h, int):
                    rt.sync(h)
                if r >= 2:
                    ts[name].append(e0.elapsed_time(e1) * 1e3)
    clocks = clk.summary()
    flop = 2.0 * M ** 3
    cub = float(np.median(ts["cublas"]))
    for name, v in ts.items():
        us = float(np.median(v))
        print(json.dumps({"gemm": f"{M}^3 bf16", "variant": name, "us_p50": round(us, 2), "us_min": round(min(v), 2),
                          "tflops": round(flop / us / 1e6, 1), "vs_cublas": round(cub / us, 3), "clocks": clocks}),
              flush=True)
    rt.close()


def run_sustained(torch, rt, variants, s, M, seconds):
    """Power-capped steady state: each variant back to back for `seconds` (launches queued in
    batches, CUDA events around each batch), rounds interleaved; NVML energy and SM clock over
    each variant's window. One JSON line per variant and round."""
    import pynvml as N
    N.nvmlInit()
    nv = N.nvmlDeviceGetHandleByIndex(torch.cuda.current_device())
    flop = 2.0 * M ** 3
    for fn in variants.values():                      # warm every variant once
        h = fn()
        if isinstance(h, int):
            rt.sync(h)
    torch.cuda.synchronize()
    batch = 16
    for rnd in range(int(os.environ.get("GEMM_ROUNDS", "2"))):
        for name, fn in variants.items():
            hs, n, tot_ms, clks = [], 0, 0.0, []
            e_j0 = N.nvmlDeviceGetTotalEnergyConsumption(nv)
            while tot_ms < seconds * 1e3:
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                for _ in range(batch):
                    h = fn()
                    if isinstance(h, int):
                        hs.append(h)
                e1.record(s)
                e1.synchronize()
                for h in hs:
                    rt.sync(h)
                hs.clear()
                tot_ms += e0.elapsed_time(e1)
                n += batch
                clks.append(N.nvmlDeviceGetClockInfo(nv, N.NVML_CLOCK_SM))
            e_j = (N.nvmlDeviceGetTotalEnergyConsumption(nv) - e_j0) / 1e3
            us = tot_ms * 1e3 / n
            print(json.dumps({"gemm": f"{M}^3 bf16", "mode": "sustained", "round": rnd, "variant": name,
                              "launches": n, "us_mean": round(us, 2), "tflops": round(flop / us / 1e6, 1),
                              "joules_per_gemm": round(e_j / n, 4), "sm_mhz_median": float(np.median(clks))}),
                  flush=True)
    rt.close()


if __name__ == "__main__":
    main()
