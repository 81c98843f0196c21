#!/bin/bash
# Final evidence (round 2 end): GPU suite, smoke, default bench line (20 steps, as the driver),
# reference arm, gemm pair in-tile victim, the scale dry run for N = 2 on one GPU (shared-GPU gloo)
mkdir -p gpurun_out/r02z
export FLEP_EVIDENCE_DIR=gpurun_out/r02z
timeout 2000 python -m pytest tests -m gpu -q > gpurun_out/r02z/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/r02z/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/r02z/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/r02z/smoke.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r02z/bench.json 2> gpurun_out/r02z/bench.err; echo "bench rc=$?"
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/r02z/ref.json 2> gpurun_out/r02z/ref.err; echo "ref rc=$?"
python - <<'PY'
import json
d = json.loads(open("gpurun_out/r02z/bench.json").read().strip().splitlines()[-1])
print("value", d["value"], "e2e", d["e2e"]["value"], "frac", d["roofline"]["frac"], "clocks", d["clocks"])
print({k: (v.get("overhead_pct"), v.get("overhead_ci95_pct")) for k, v in d["kernels"].items() if isinstance(v, dict)})
print("op2", json.dumps(d.get("operating_points") or d.get("op2"))[:400])
subs = d.get("configs") or {}
print("subs", list(subs.keys()) if isinstance(subs, dict) else subs)
r = json.loads(open("gpurun_out/r02z/ref.json").read().strip().splitlines()[-1])
print("ref", r["value"], r["ms_per_step"])
PY
