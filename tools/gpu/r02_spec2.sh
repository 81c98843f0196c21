#!/bin/bash
# speculative fetch in the plain counter worker (R34): overhead A/B and the GPU tests
mkdir -p gpurun_out/r02spec
timeout 900 python -m pytest tests/test_gpu_spec_fetch.py -x -q 2>&1 | tail -3
CASES=spmv:1:1,spmv:1:1:0:0:0:0:0:0:1,spmv:1:1:0:0:0:0:0:0:1:1,spmv:2:1,spmv:2:1:0:0:0:0:0:0:1,spmv:2:1:0:0:0:0:0:0:1:1
for r in 1 2; do
timeout 600 python tools/ab_overhead.py $CASES > gpurun_out/r02spec/ab_spec2_$r.jsonl 2>&1
python -c "
import json,sys
for l in open('gpurun_out/r02spec/ab_spec2_$r.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print(d['case'], d['wrapped_us'], d['unwrapped_us'], d['overhead_pct'], d['worker_span_us'])
"
done
