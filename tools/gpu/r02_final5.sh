#!/bin/bash
# Final validation after R38: the whole GPU suite, smoke, the default bench line and the reference arm.
mkdir -p gpurun_out/f6
rm -f gpurun_out/f6/*
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/f6/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/f6/pytest_gpu.log
tail -3 gpurun_out/f6/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/f6/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/f6/smoke.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/f6/bench.json 2> gpurun_out/f6/bench.err; echo "bench rc=$?"
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/f6/ref.json 2> gpurun_out/f6/ref.err; echo "ref rc=$?"
python - <<'PY'
import json
d = json.loads(open("gpurun_out/f6/bench.json").read().strip().splitlines()[-1])
print("value", d["value"], "e2e", d["e2e"]["value"], "frac", d["roofline"]["frac"], "clocks", d["clocks"])
print("ovh", d["wrapper_overhead_pct"], "parity", d["parity"]["ok"])
r = json.loads(open("gpurun_out/f6/ref.json").read().strip().splitlines()[-1])
print("ref", r["value"], r["ms_per_step"])
PY
