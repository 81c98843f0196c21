#!/bin/bash
# R38 selection rule: ring form up to K = 1 (default), 2 or 4, on the K = 2 and K = 4 cases.
mkdir -p gpurun_out/ringk
CS=stencil:1:2:0:1,stencil:1:4:0:1,spmvvec:1:2:0:1
for r in 1 2 3; do
  for v in k1 k2 k4; do
    FLEP_LIB_PATH=$PWD/build_variants/$v.so timeout 300 python tools/ab_overhead.py $CS 2>> gpurun_out/ringk/ab.err | grep '^{' | \
      python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); print(json.dumps({'ring_max_k':'$v','round':$r,'case':d['case'],'wrapped_us':d['wrapped_us'],'unwrapped_us':d['unwrapped_us'],'overhead_pct':d['overhead_pct']}))
"
  done
done | tee gpurun_out/ringk/ab.jsonl
