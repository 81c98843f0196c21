#!/bin/bash
# SpMV body occupancy / gathers-in-flight variants: worker C = 1 / C = 2 (speculative fetch) vs unwrapped
mkdir -p gpurun_out/r02occ
CASES=spmv:1:1:0:0:0:0:0:0:1,spmv:2:1:0:0:0:0:0:0:1
for rep in 1 2; do
for v in base m6u6 m6u8 m7u6; do
  FLEP_LIB_PATH=build_variants/$v.so timeout 300 python tools/ab_overhead.py $CASES >> gpurun_out/r02occ/ab.jsonl 2>> gpurun_out/r02occ/ab.err
done
done
python - <<'PY'
import json
for l in open("gpurun_out/r02occ/ab.jsonl"):
    if l.startswith("{"):
        d = json.loads(l); print(d["lib"], d["case"], d["wrapped_us"], d["unwrapped_us"], d["overhead_pct"])
PY
