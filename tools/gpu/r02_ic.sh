#!/bin/bash
mkdir -p gpurun_out/r02ic
timeout 900 python -m pytest tests/test_gpu_in_chunk.py -x -q > gpurun_out/r02ic/pytest.log 2>&1; echo "pytest rc=$?"; tail -30 gpurun_out/r02ic/pytest.log
timeout 300 python tools/ab_overhead.py spmv:1:1,spmv:2:1:0:0:0:1,spmv:4:1:0:0:0:1,spmv:8:1:0:0:0:1,spmvvec:4:1:0:0:0:1,spmvvec:8:1:0:0:0:1,stencil:2:1:0:0:0:1,stencil:4:1:0:0:0:1,stencil:8:1:0:0:0:1 > gpurun_out/r02ic/ab.jsonl 2>&1
cut -c1-200 gpurun_out/r02ic/ab.jsonl
