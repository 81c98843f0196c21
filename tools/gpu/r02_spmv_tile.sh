#!/bin/bash
# SpMV CSR-stream tile / U variants: worker C = 1 and C = 2 (speculative fetch) vs unwrapped
mkdir -p gpurun_out/r02st
for rep in 1 2; do
for v in base tile4096 u6 tile4096_u6; do
  FLEP_LIB_PATH=build_variants/$v.so timeout 300 python tools/ab_overhead.py spmv:1:1:0:0:0:0:0:0:1,spmv:2:1:0:0:0:0:0:0:1 >> gpurun_out/r02st/ab.jsonl 2>> gpurun_out/r02st/ab.err
done
done
python - <<'PY'
import json
for l in open("gpurun_out/r02st/ab.jsonl"):
    d = json.loads(l)
    print(d["lib"], d["case"], d["wrapped_us"], d["unwrapped_us"], d["overhead_pct"])
PY
tail -2 gpurun_out/r02st/ab.err
