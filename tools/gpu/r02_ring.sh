#!/bin/bash
# R38: CLC worker without the per-block CTA barrier (mbarrier response ring) vs the barrier form,
# stencil 4096^2 (the configs[1] waiting kernel: CLC C = 1, K = 4; also K = 1 and C = 2), the
# SAXPY / SpMV-vector warp-task bodies with CLC; then the CLC / stencil GPU tests on the ring build.
mkdir -p gpurun_out/ring
CS=stencil:1:4:0:1,stencil:1:1:0:1,stencil:2:2:0:1,spmvvec:1:1:0:1,spmvvec:2:2:0:1
for r in 1 2 3; do
  for v in ring noring; do
    FLEP_LIB_PATH=$PWD/build_variants/$v.so timeout 300 python tools/ab_overhead.py $CS 2>> gpurun_out/ring/ab.err | grep '^{' | \
      python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); print(json.dumps({'lib':'$v','round':$r,'case':d['case'],'wrapped_us':d['wrapped_us'],'unwrapped_us':d['unwrapped_us'],'overhead_pct':d['overhead_pct']}))
"
  done
done | tee gpurun_out/ring/ab.jsonl
timeout 900 python -m pytest tests/test_gpu_clc.py tests/test_gpu_parity.py -x -q 2>&1 | tail -2
