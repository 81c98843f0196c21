#!/bin/bash
# full check after the R35 change: GPU suite, smoke, default bench line
mkdir -p gpurun_out/r02f2
export FLEP_EVIDENCE_DIR=gpurun_out/r02f2
[ -n "$SKIP_TESTS" ] || timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r02f2/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -4 gpurun_out/r02f2/pytest_gpu.log
[ -n "$SKIP_TESTS" ] || timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02f2/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/r02f2/smoke.log
start=$(date +%s); timeout 900 python bench.py > gpurun_out/r02f2/bench.json 2> gpurun_out/r02f2/bench.err; echo "bench rc=$?"
echo "bench wall $(( $(date +%s) - start )) s"
python - <<'PY'
import json
d = json.loads(open("gpurun_out/r02f2/bench.json").read().strip().splitlines()[-1])
print({k: d.get(k) for k in ("value", "unit", "ms_per_step", "gpu_launches")})
print("roofline", d.get("roofline"))
print("e2e", {k: d["e2e"].get(k) for k in ("value", "unit")})
print("overhead", d.get("wrapper_overhead_pct"))
e13 = d.get("configs", {}).get("E13_never_preempted", {})
print("gemm", e13.get("gemm_2sm_8192"))
print("wall", d.get("configs", {}).get("wall_s"))
PY
