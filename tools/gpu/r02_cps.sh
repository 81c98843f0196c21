#!/bin/bash
# Victim occupancy sweep (configs[1]): resident SpMV workers per SM k = 8 (occupancy), 7, 6, 5, 4.
# Fewer workers per SM share the SM's gather interface among fewer blocks, so each block (the
# preemption granularity) finishes sooner; the question is what the SpMV's throughput pays.
mkdir -p gpurun_out/cps
for r in 1 2; do
for k in 0 7 6 5 4; do
  timeout 300 python bench.py --steps 20 --warmup 5 --sub 0 --op2 0 --lp-cps $k > gpurun_out/cps/k${k}_r$r.json 2> gpurun_out/cps/k${k}_r$r.err
  python - "$k" "$r" <<'PY'
import json, sys
d = json.loads(open(f"gpurun_out/cps/k{sys.argv[1]}_r{sys.argv[2]}.json").read().strip().splitlines()[-1])
s = d["kernels"]["spmv"]
print(json.dumps({"lp_cps": d["config"]["lp_ctas_per_sm"], "round": int(sys.argv[2]), "drain_p50": d["drain_us"]["p50"],
                  "drain_p99": d["drain_us"]["p99"], "chunk_us": d["latency_budget"]["victim_chunk_us"],
                  "spmv_wrapped_us": s["wrapped_us"], "spmv_unwrapped_us": s["unwrapped_us"],
                  "spmv_overhead_pct": s["overhead_pct"], "e2e_us": d["e2e"]["value"], "frac": d["roofline"]["frac"],
                  "sm_mhz": d["clocks"].get("sm_mhz"), "parity_ok": d["parity"]["ok"]}))
PY
done; done | tee gpurun_out/cps/summary.jsonl
