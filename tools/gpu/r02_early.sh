#!/bin/bash
# R36 early step: GPU tests of the speculative-fetch worker, then an interleaved A/B of the SpMV
# victim with and without the early step (same source, -DFLEP_NO_EARLY_STEP), two rounds
mkdir -p gpurun_out/r02early
timeout 1200 python -m pytest -x -q tests/test_gpu_spec_fetch.py tests/test_gpu_parity.py > gpurun_out/r02early/tests.log 2>&1
rc=$?; echo "tests rc=$rc"; tail -3 gpurun_out/r02early/tests.log
[ $rc -eq 0 ] || exit 1
for rep in 1 2; do
for v in early noearly; do
  FLEP_LIB_PATH=build_variants/$v.so timeout 300 python tools/ab_overhead.py spmv:1:1:0:0:0:0:0:0:1,spmv:1:1,spmv:2:1:0:0:0:0:0:0:1 >> gpurun_out/r02early/ab.jsonl 2>> gpurun_out/r02early/ab.err
done
done
python - <<'PY'
import json
for l in open("gpurun_out/r02early/ab.jsonl"):
    if l.startswith("{"):
        d = json.loads(l); print(d["lib"], d["case"], d["wrapped_us"], d["unwrapped_us"], d["overhead_pct"])
PY
tail -2 gpurun_out/r02early/ab.err
