"""DES prediction vs the B200 measurement for the configs[3] queue (SURVEY §8(c) O3 simulate mode,
§8(d) C4 "DES-predicted vs measured ANTT"). Test infrastructure (it imports the oracle, so it
lives under tests/; run by tests/test_oracle_des.py, or directly to print the report).

Input: the per-kernel record of one queue run (tests/golden/queue_debug_r02.json: name, host
arrival, first start, finish, epochs, standalone time, per policy) and that run's measured ANTT.
The simulation replays the FIFO run's arrival times with the measured standalone times as both
T_e and T_true, the queue's overhead estimate O, a drain d (the measured preemption latency) and a
start delay s (the measured launch-to-start gap), and prints predicted vs measured ANTT per policy.
"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle import des  # noqa: E402
from oracle import metrics  # noqa: E402


def predict(debug, overhead_ns=20_000, drain_ns=12_000, start_ns=15_000, slice_blocks_ns=None):
    fifo = debug["FIFO"]
    ks = []
    for i, (name, arr, st, fin, ep, alone) in enumerate(fifo):
        ks.append(des.KernelSpec(i, int(arr), 0, int(alone), int(overhead_ns), int(alone)))
    out = {}
    for kind in (des.FIFO, des.HPF, des.REORDER):
        r = des.simulate(kind, ks, des.SimParams(drain_ns=drain_ns, start_ns=start_ns))
        tt = [r.turnaround[k.id] for k in ks]
        out[kind] = metrics.antt(tt, [k.t_true for k in ks])
    return out


def main():
    g = os.path.join(ROOT, "tests", "golden")
    debug = json.load(open(os.path.join(g, "queue_debug_r02.json")))
    meas = json.load(open(os.path.join(g, "queue_measured_r02.json")))
    # start delay: the median gap between a FIFO kernel's host arrival and its first start when the
    # GPU was idle (arrival after the previous finish)
    fifo = sorted(debug["FIFO"], key=lambda r: r[1])
    gaps, prev = [], 0
    for name, arr, st, fin, ep, alone in fifo:
        if arr > prev:
            gaps.append(st - arr)
        prev = max(prev, fin)
    start_ns = int(np.median(gaps)) if gaps else 15_000
    pred = predict(debug, overhead_ns=meas["overhead_estimate_ns"], start_ns=start_ns)
    rows = {k: {"predicted_antt": round(v, 3), "measured_antt": meas["antt"][k],
                "ratio": round(v / meas["antt"][k], 3)} for k, v in pred.items()}
    out = {"what": "oracle DES simulate mode vs the B200 configs[3] run (same arrivals, measured standalone times)",
           "start_delay_ns": start_ns, "drain_ns": 12_000, "overhead_ns": meas["overhead_estimate_ns"],
           "policies": rows,
           "natt_gain_hpf_vs_fifo": {"predicted": round(pred[des.FIFO] / pred[des.HPF], 3),
                                     "measured": round(meas["antt"]["FIFO"] / meas["antt"]["HPF"], 3)}}
    print(json.dumps(out))
    return out


if __name__ == "__main__":
    main()
