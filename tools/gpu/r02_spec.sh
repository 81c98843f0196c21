#!/bin/bash
# speculative fetch (R34): plain C=1 worker vs the in-chunk worker at C=1 with the speculative
# fetch (poll + fetch in one round trip), and the in-chunk worker without it (experiment build)
mkdir -p gpurun_out/r02spec
CASES=spmv:1:1,spmv:1:1:0:0:0:1,spmvvec:1:1,spmvvec:1:1:0:0:0:1,stencil:1:1,stencil:1:1:0:0:0:1,spmv:2:1,spmv:2:1:0:0:0:1
timeout 600 python tools/ab_overhead.py $CASES > gpurun_out/r02spec/ab_spec.jsonl 2>&1
FLEP_LIB_PATH=$PWD/build_variants/nospec.so timeout 600 python tools/ab_overhead.py $CASES > gpurun_out/r02spec/ab_nospec.jsonl 2>&1
for f in gpurun_out/r02spec/ab_*.jsonl; do echo "== $f"; python -c "
import json,sys
for l in open('$f'):
    if l.startswith('{'):
        d=json.loads(l); print(d['case'], d['wrapped_us'], d['unwrapped_us'], d['overhead_pct'], d['worker_span_us'])
"; done
timeout 900 python -m pytest tests/test_gpu_in_chunk.py -x -q 2>&1 | tail -2
