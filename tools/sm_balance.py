import json, os, sys
import numpy as np
sys.path.insert(0, os.getcwd())
from synth import gen
import torch
from paper_conf_asplos_wulzj17_b200 import flep as F
from bench import L2Flush
rt = F.Runtime(exec_on_user_stream=True)
flush = L2Flush(torch)
T = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()
rp, col, val, x = gen.csr_inputs(1 << 20, seed=2)
dev = [T(rp), T(col), T(val), T(x)]
y = torch.zeros(1 << 20, device="cuda")
args = F.spmv_args(y, *dev)
out = {}
for name, kw in (("counter", {}), ("spec", {"spec_fetch": True})):
    k = rt.register_kernel(F.BODY_SPMV_CSR_F32, chunk=1, poll=1, **kw)
    per_sm = []
    exits = []
    for rep in range(10):
        flush.zero_(); torch.cuda.synchronize()
        h = rt.launch(k, F.spmv_grid(1 << 20), args, stream=torch.cuda.current_stream())
        rt.sync(h)
        ev = [e for e in rt.events(h, 1) if e.t_entry > 0]
        t0 = min(e.t_entry for e in ev)
        sm = np.zeros(rt.num_sms)
        for e in ev: sm[e.smid] += e.n_blocks
        per_sm.append(sm)
        exits.append(sorted((e.t_exit - t0) / 1e3 for e in ev))
    S = np.mean(per_sm, axis=0)
    ex = np.array(exits)
    out[name] = {"blocks_per_sm_mean": float(S.mean()), "min": float(S.min()), "max": float(S.max()), "std": float(S.std()),
                 "cv_pct": float(100 * S.std() / S.mean()), "corr_between_reps": float(np.corrcoef(per_sm[0], per_sm[1])[0, 1]),
                 "exit_first_us": float(np.median(ex[:, 0])), "exit_p10_us": float(np.median(ex[:, len(ev)//10])),
                 "exit_p50_us": float(np.median(ex[:, len(ev)//2])), "exit_last_us": float(np.median(ex[:, -1])),
                 "slowest_sms": [int(i) for i in np.argsort(S)[:8]], "fastest_sms": [int(i) for i in np.argsort(S)[-8:]]}
print(json.dumps(out))
rt.close()
