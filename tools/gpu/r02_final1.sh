#!/bin/bash
# smoke, the default bench line (with the C = 2 operating point), the reference arm
mkdir -p gpurun_out/r02f
export FLEP_EVIDENCE_DIR=gpurun_out/r02f
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02f/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/r02f/smoke.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r02f/bench.json 2> gpurun_out/r02f/bench.err; echo "bench rc=$?"; tail -c 600 gpurun_out/r02f/bench.err
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/r02f/ref.json 2> gpurun_out/r02f/ref.err; echo "ref rc=$?"
python - <<'PY'
import json
d = json.loads(open("gpurun_out/r02f/bench.json").read().strip().splitlines()[-1])
print("value", d["value"], "e2e", d["e2e"]["value"], "ovh", d["wrapper_overhead_pct"], "frac", d["roofline"]["frac"])
print(json.dumps(d["operating_points"]))
print(d["configs"]["wall_s"])
r = json.loads(open("gpurun_out/r02f/ref.json").read().strip().splitlines()[-1])
print("ref", r["value"], r["ms_per_step"])
PY
