"""Fixed per-launch cost: wrapped vs unwrapped SAXPY at tiny and medium sizes (CUDA events)."""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    from paper_conf_asplos_wulzj17_b200 import build, flep as F
    build.build()
    rt = F.Runtime(exec_on_user_stream=True)
    s = torch.cuda.current_stream()
    for n in (256, 256 * 148, 1 << 20, 1 << 24):
        x = torch.ones(n, dtype=torch.int32, device="cuda")
        y = torch.ones(n, dtype=torch.int32, device="cuda")
        a = F.saxpy_i32_args(y, x, 3)
        k = rt.register_kernel(F.BODY_SAXPY_I32, chunk=8, poll=1)
        res = {}
        for mode in ("unwrapped", "wrapped", "wrapped_b2b", "unwrapped_b2b"):
            ts = []
            for r in range(30):
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                reps = 10 if mode.endswith("b2b") else 1
                hs = []
                for _ in range(reps):
                    if mode.startswith("wrapped"):
                        hs.append(rt.launch(k, F.saxpy_grid(n), a, stream=s))
                    else:
                        rt.launch_unwrapped(F.BODY_SAXPY_I32, F.saxpy_grid(n), a, stream=s)
                e1.record(s)
                e1.synchronize()
                for h in hs:
                    rt.sync(h)
                if r >= 5:
                    ts.append(e0.elapsed_time(e1) * 1e3 / reps)
            res[mode] = round(float(np.median(ts)), 2)
        print(json.dumps({"n": n, **res}), flush=True)
    rt.close()


if __name__ == "__main__":
    main()
