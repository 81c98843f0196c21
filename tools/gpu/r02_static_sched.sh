#!/bin/bash
# R37 static schedule: GPU tests (new + the spec-fetch / parity / runtime suites), then the A/B:
# the default victim cases against the previous library (regression), and the static cases
mkdir -p gpurun_out/r02r37
timeout 1800 python -m pytest -x -q tests/test_gpu_static_sched.py tests/test_gpu_spec_fetch.py tests/test_gpu_parity.py tests/test_gpu_runtime.py > gpurun_out/r02r37/tests.log 2>&1
rc=$?; echo "tests rc=$rc"; tail -4 gpurun_out/r02r37/tests.log
[ $rc -eq 0 ] || exit 1
BASE=spmv:1:1:0:0:0:0:0:0:1,spmv:2:1:0:0:0:0:0:0:1,stencil:1:4:0:1
STAT=stencil:1:1:0:0:0:0:0:1:0:1,stencil:1:2:0:0:0:0:0:1:0:1,stencil:2:1:0:0:0:0:0:1:0:1,stencil:1:1:0:0:0:0:0:0:0:1,stencil:1:1:0:0:0:0:1,spmv:2:1:0:0:0:0:0:1:0:1,spmv:1:1:0:0:0:0:1
for rep in 1 2; do
  FLEP_LIB_PATH=build_variants/base.so timeout 300 python tools/ab_overhead.py $BASE >> gpurun_out/r02r37/ab.jsonl 2>> gpurun_out/r02r37/ab.err
  FLEP_LIB_PATH=build_variants/r37.so timeout 300 python tools/ab_overhead.py $BASE,$STAT >> gpurun_out/r02r37/ab.jsonl 2>> gpurun_out/r02r37/ab.err
done
python - <<'PY'
import json
for l in open("gpurun_out/r02r37/ab.jsonl"):
    if l.startswith("{"):
        d = json.loads(l); print(d["lib"], d["case"], d["wrapped_us"], d["unwrapped_us"], d["overhead_pct"])
PY
tail -2 gpurun_out/r02r37/ab.err
