#!/bin/bash
mkdir -p gpurun_out/r02q
export FLEP_EVIDENCE_DIR=gpurun_out/r02q
timeout 300 python bench.py --config queue > gpurun_out/r02q/queue_alone.json 2> gpurun_out/r02q/queue_alone.err; echo "rc=$?"
cp gpurun_out/r02q/queue_debug.json gpurun_out/r02q/queue_debug_alone.json
timeout 600 python bench.py --steps 20 --warmup 5 --skip-sub "configs[4]" > gpurun_out/r02q/bench.json 2> gpurun_out/r02q/bench.err; echo "rc=$?"
python - <<'PY'
import json
a = json.loads(open("gpurun_out/r02q/queue_alone.json").read().strip().splitlines()[-1])
print("alone", a["antt"], a["makespan_ms"], a["launch_call_us"])
d = json.loads(open("gpurun_out/r02q/bench.json").read().strip().splitlines()[-1])
c = d["configs"]["configs[3]"]
print("sub", c["antt"], c["makespan_ms"], c["launch_call_us"])
PY
