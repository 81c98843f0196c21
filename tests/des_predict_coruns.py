"""DES prediction vs the B200 co-run matrices (bench.py --config coruns; E4 / E6 / E8, Figs. 8, 10,
12): the oracle DES simulate mode on each case's nominal arrivals (0, 20, 40 µs),
priorities and the measured standalone times (tests/golden/coruns_measured_r02.json), with the
runtime's overhead estimate O, a drain d and a start delay s. Test infrastructure (imports the
oracle; run by tests/test_oracle_des.py, or directly to print the report)."""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle import des  # noqa: E402
from oracle import metrics  # noqa: E402

sys.path.insert(0, ROOT)
import bench_configs  # noqa: E402  (the case list only: no GPU code runs on import)


def predict(meas, drain_ns=12_000, start_ns=9_000):
    t_alone = {k: int(v * 1e3) for k, v in meas["t_alone_us"].items()}
    overhead = meas["config"]["overhead_estimate_ns"]
    rows = []
    for exp, name, trace in bench_configs.corun_cases():
        ks = [des.KernelSpec(j["id"], j["arrival_ns"], j["priority"], t_alone[f"{j['type']}-{j['size_class']}"],
                             overhead, t_alone[f"{j['type']}-{j['size_class']}"]) for j in trace]
        p = des.SimParams(drain_ns=drain_ns, start_ns=start_ns)
        sim = {kind: des.simulate(kind, ks, p) for kind in (des.FIFO, des.HPF)}
        tt = {kind: [r.turnaround[k.id] for k in ks] for kind, r in sim.items()}
        al = [k.t_true for k in ks]
        row = {"exp": exp, "case": name}
        if exp == "E4":
            row["pred"] = tt[des.FIFO][1] / tt[des.HPF][1]
        else:
            row["pred"] = metrics.antt(tt[des.FIFO], al) / metrics.antt(tt[des.HPF], al)
        rows.append(row)
    return rows


def main():
    meas = json.load(open(os.path.join(ROOT, "tests", "golden", "coruns_measured_r02.json")))
    got = {(r["exp"], r["case"]): r.get("hp_speedup", r.get("antt_gain")) for r in meas["cases"]}
    rows = predict(meas)
    for r in rows:
        r["measured"] = got[(r["exp"], r["case"])]
        r["ratio"] = round(r["pred"] / r["measured"], 3)
        r["pred"] = round(r["pred"], 3)
    summ = {exp: {"pred_mean": round(float(np.mean([r["pred"] for r in rows if r["exp"] == exp])), 3),
                  "meas_mean": round(float(np.mean([r["measured"] for r in rows if r["exp"] == exp])), 3),
                  "ratio_min": min(r["ratio"] for r in rows if r["exp"] == exp),
                  "ratio_max": max(r["ratio"] for r in rows if r["exp"] == exp)} for exp in ("E4", "E6", "E8")}
    out = {"what": "oracle DES simulate mode vs the B200 co-run matrices (nominal arrivals, measured standalone "
                   "times, O from the run, drain 12 us, start 9 us)", "summary": summ, "cases": rows}
    print(json.dumps(out))
    return out


if __name__ == "__main__":
    main()
