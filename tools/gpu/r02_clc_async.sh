#!/bin/bash
# CLC worker with the async poll (R22 on the CLC fetch): stencil 4096^2 overhead, and the CLC tests
mkdir -p gpurun_out/r02clc
timeout 900 python -m pytest tests/test_gpu_clc.py -x -q 2>&1 | tail -2
CS=stencil:1:4:0:1,stencil:1:4:0:1:0:0:0:1,stencil:1:1:0:1,stencil:1:1:0:1:0:0:0:1,stencil:2:2:0:1,stencil:2:2:0:1:0:0:0:1
for r in 1 2; do
timeout 600 python tools/ab_overhead.py $CS > gpurun_out/r02clc/ab_$r.jsonl 2>&1
python -c "
import json
for l in open('gpurun_out/r02clc/ab_$r.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print(d['case'], d['wrapped_us'], d['unwrapped_us'], d['overhead_pct'])
"
done
