"""Wrapper overhead of a user-defined body (include/flep_body.cuh; the example
tests/user_body/body_affine_rev.cu): the FLEP worker at several chunk sizes, the CLC worker and the
static persistent twin against the original grid, interleaved and dithered, L2 flushed; plus the
full-GPU drain of the worker (device self-trigger at a random block). One JSON line."""
import ctypes as C
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from synth import gen  # noqa: E402

PER = 512


class AffineRevArgs(C.Structure):
    _fields_ = [("y", C.c_void_p), ("x", C.c_void_p), ("a", C.c_int32), ("c", C.c_int32), ("n", C.c_uint32)]


def main():
    import torch
    from paper_conf_asplos_wulzj17_b200 import build, flep as F
    from paper_conf_asplos_wulzj17_b200.calibrate import event_mean_us
    from bench import L2Flush
    build.build()
    lib = build.build_user_body(os.path.join(ROOT, "tests", "user_body", "body_affine_rev.cu"),
                                os.path.join(ROOT, "tests", "user_body", "build", "libaffine_rev.so"))
    rt = F.Runtime(exec_on_user_stream=True)
    body = rt.register_body(lib, "affine_rev")
    n = 1 << 26                                        # 256 MiB in + out: ~80 us at HBM speed
    x, _ = gen.saxpy_i32_inputs(n, seed=5)
    xd = torch.from_numpy(x).cuda()
    yd = torch.empty(n, dtype=torch.int32, device="cuda")
    args = AffineRevArgs(yd.data_ptr(), xd.data_ptr(), 3, 7, n)
    grid = (-(-n // PER), 1, 1)
    flush = L2Flush(torch)
    s = torch.cuda.current_stream()
    ks = {f"flep_c{c}": rt.register_kernel(body, chunk=c, poll=1) for c in (1, 4, 16, 64)}
    ks.update({f"flep_spec_c{c}": rt.register_kernel(body, chunk=c, poll=1, spec_fetch=True) for c in (1, 16, 64)})
    ks["clc_c1_k4"] = rt.register_kernel(body, chunk=1, poll=4, clc=True)
    variants = {"unwrapped": lambda: rt.launch_unwrapped(body, grid, args, stream=s),
                "static_c4": lambda: rt.launch_static(body, grid, args, chunk=4, stream=s)}
    for name, k in ks.items():
        variants[name] = (lambda k=k: rt.launch(k, grid, args, stream=s))
    ts = {v: [] for v in variants}
    for r in range(24):
        for name, fn in variants.items():
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            h = fn()
            e1.record(s)
            e1.synchronize()
            if isinstance(h, int):
                rt.sync(h)
            if r >= 4:
                ts[name].append(e0.elapsed_time(e1) * 1e3)
    u = event_mean_us(ts["unwrapped"])
    cps, w = rt.workers_for(body)
    out = {"workers": w, "ctas_per_sm": cps, "what": "user-defined body affine_rev (int32 y = a*x[mirror] + c*block, 512 elements per block, "
                   "2^26 elements), CUDA-event means of 20 interleaved reps, L2 flushed",
           "unwrapped_us": round(u, 2), "gbs_unwrapped": round(8 * n / u / 1e3, 1)}
    for name in variants:
        if name != "unwrapped":
            v = event_mean_us(ts[name])
            out[name + "_us"] = round(v, 2)
            out[name + "_overhead_pct"] = round((v / u - 1) * 100, 2)
    # drain: device self-trigger at a random block of the C = 1 worker, temporal
    rt2 = F.Runtime(coverage=False)
    body2 = rt2.register_body(lib, "affine_rev")
    k2 = rt2.register_kernel(body2, chunk=1, poll=1)
    g = gen.rng(11)
    lat = []
    for i in range(12):
        rt2.arm_next_trigger(int(g.integers(grid[0] // 4, 3 * grid[0] // 4)), rt2.num_sms)
        h = rt2.launch(k2, grid, args)
        rt2.wait_epoch(h, timeout_ns=20_000_000_000)
        if rt2.query(h).state == F.STATE_PREEMPTED:
            ep = rt2.epoch_info(h, 1)
            lat.append((ep.t_end - ep.t_trigger) / 1e3)
            rt2.resume(h)
        rt2.sync(h, timeout_ns=20_000_000_000)
    torch.cuda.synchronize()
    out["drain_us_p50_c1"] = round(float(np.median(lat)), 2) if lat else None
    ref_ok = True
    xx = x.astype(np.int64)
    nb = grid[0]
    mir = np.concatenate([xx, np.zeros(nb * PER - n, dtype=np.int64)]).reshape(nb, PER)[:, ::-1].reshape(-1)[:n]
    ref = ((3 * mir + 7 * (np.arange(n) // PER)) & 0xFFFFFFFF).astype(np.uint32).view(np.int32)
    ref_ok = bool(np.array_equal(yd.cpu().numpy(), ref))
    out["result_exact"] = ref_ok
    print(json.dumps(out))
    rt.close()
    rt2.close()


if __name__ == "__main__":
    main()
