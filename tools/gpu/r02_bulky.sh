#!/bin/bash
# experiment: SpMV y through shared memory + bulk copy (WAR-on-store-register hypothesis)
mkdir -p gpurun_out/r02bulky
CS=spmv:1:1:0:0:0:0:0:0:1,spmv:2:1:0:0:0:0:0:0:1,spmv:1:1:0:0:0:0:0:1
for v in default bulky default bulky; do
  if [ $v = default ]; then unset FLEP_LIB_PATH; else export FLEP_LIB_PATH=$PWD/build_variants/$v.so; fi
  timeout 600 python tools/ab_overhead.py $CS > gpurun_out/r02bulky/ab_$v.jsonl 2>&1
  python -c "
import json
for l in open('gpurun_out/r02bulky/ab_$v.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print('$v', d['case'], d['wrapped_us'], d['unwrapped_us'], d['overhead_pct'])
"
done
FLEP_LIB_PATH=$PWD/build_variants/bulky.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k spmv 2>&1 | tail -1
