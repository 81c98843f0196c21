#!/bin/bash
# what a per-chunk poll adds to the static persistent twin (no fetch): sync poll (1) / async (2)
mkdir -p gpurun_out/r02sp
CASES=stencil:1:1:0:0:0:0:1,spmv:1:1:0:0:0:0:1,spmv:2:1:0:0:0:0:1,stencil:1:4:0:1
for rep in 1 2; do
for v in base spoll1 spoll2; do
  FLEP_LIB_PATH=build_variants/$v.so timeout 300 python tools/ab_overhead.py $CASES >> gpurun_out/r02sp/ab.jsonl 2>> gpurun_out/r02sp/ab.err
done
done
python - <<'PY'
import json
for l in open("gpurun_out/r02sp/ab.jsonl"):
    if l.startswith("{"):
        d = json.loads(l); print(d["lib"], d["case"], d["wrapped_us"], d["unwrapped_us"], d["overhead_pct"])
PY
tail -2 gpurun_out/r02sp/ab.err
