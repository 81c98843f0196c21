#!/bin/bash
# R36 in-body stop for the SpMV (in-chunk worker with the decision on the body's barrier)
mkdir -p gpurun_out/r02ibs
timeout 900 python -m pytest tests/test_gpu_in_chunk.py -x -q 2>&1 | tail -2
CS=spmv:1:1:0:0:0:0:0:0:1,spmv:2:1:0:0:0:0:0:0:1,spmv:2:1:0:0:0:1,spmv:4:1:0:0:0:1,spmv:8:1:0:0:0:1,spmv:4:1
for r in 1 2; do
timeout 600 python tools/ab_overhead.py $CS > gpurun_out/r02ibs/ab_$r.jsonl 2>&1
python -c "
import json
for l in open('gpurun_out/r02ibs/ab_$r.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print(d['case'], d['wrapped_us'], d['unwrapped_us'], d['overhead_pct'])
"
done
