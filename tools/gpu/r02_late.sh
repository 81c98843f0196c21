#!/bin/bash
# R35 late scheduling point: A/B against the previous commit's library and a build without the hook
mkdir -p gpurun_out/r02late
C1=spmv:1:1,spmv:1:1:0:0:0:0:0:0:1,spmv:2:1:0:0:0:0:0:0:1
C2=$C1,spmv:1:1:0:0:0:0:0:0:1:1,spmv:2:1:0:0:0:0:0:0:1:1
for v in base nohook cur; do
  if [ $v = cur ]; then unset FLEP_LIB_PATH; CS=$C2; else export FLEP_LIB_PATH=$PWD/build_variants/$v.so; CS=$C1; fi
  timeout 600 python tools/ab_overhead.py $CS > gpurun_out/r02late/ab_$v.jsonl 2>&1
  python -c "
import json
for l in open('gpurun_out/r02late/ab_$v.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print('$v', d['case'], d['wrapped_us'], d['unwrapped_us'], d['overhead_pct'])
"
done
