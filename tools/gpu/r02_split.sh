#!/bin/bash
# SpMV CSR-stream with two threads per row in the row sums (FLEP_SPMV_SPLIT) vs the base body:
# parity tests on the split build, then the interleaved A/B of unwrapped and workers
mkdir -p gpurun_out/r02split
FLEP_LIB_PATH=build_variants/split.so timeout 900 python -m pytest -x -q tests/test_gpu_parity.py tests/test_gpu_spec_fetch.py -k "spmv or Spmv" > gpurun_out/r02split/tests.log 2>&1
echo "tests rc=$?"; tail -2 gpurun_out/r02split/tests.log
CASES=spmv:1:1:0:0:0:0:0:0:1,spmv:2:1:0:0:0:0:0:0:1,spmv:1:1:0:0:0:0:1
for rep in 1 2; do
for v in base split; do
  FLEP_LIB_PATH=build_variants/$v.so timeout 300 python tools/ab_overhead.py $CASES >> gpurun_out/r02split/ab.jsonl 2>> gpurun_out/r02split/ab.err
done
done
python - <<'PY'
import json
for l in open("gpurun_out/r02split/ab.jsonl"):
    if l.startswith("{"):
        d = json.loads(l); print(d["lib"], d["case"], d["wrapped_us"], d["unwrapped_us"], d["overhead_pct"])
PY
