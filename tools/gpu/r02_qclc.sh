#!/bin/bash
# Queue experiment: stencil victims on the counter with speculative fetch (C = 2, K = 1; default)
# vs the barrier-free CLC worker (C = K = 1, R38), configs[3] and configs[4], two rounds each.
mkdir -p gpurun_out/qclc
for r in 1 2; do
  for v in spec clc; do
    if [ $v = clc ]; then export FLEP_QUEUE_STENCIL=clc; else unset FLEP_QUEUE_STENCIL; fi
    timeout 600 python bench.py --config queue > gpurun_out/qclc/q_${v}_$r.json 2> gpurun_out/qclc/q_${v}_$r.err
    timeout 900 python bench.py --config scale > gpurun_out/qclc/s_${v}_$r.json 2> gpurun_out/qclc/s_${v}_$r.err
    python - "$v" "$r" <<'PY'
import json, sys
v, r = sys.argv[1], sys.argv[2]
q = json.loads(open(f"gpurun_out/qclc/q_{v}_{r}.json").read().strip().splitlines()[-1])
s = json.loads(open(f"gpurun_out/qclc/s_{v}_{r}.json").read().strip().splitlines()[-1])
print(json.dumps({"stencil_fetch": v, "round": int(r), "configs3_natt_gain": q["value"], "configs3_antt": q["antt"],
                  "configs4_value": s["value"], "configs4_unit": s.get("unit"),
                  "configs4_antt": s.get("antt"), "configs4_makespan_ms": s.get("makespan_ms")}))
PY
  done
done | tee gpurun_out/qclc/summary.jsonl
