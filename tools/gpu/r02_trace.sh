#!/bin/bash
mkdir -p gpurun_out/r02ab
FLEP_LIB_PATH=build_variants/trace.so TRACE_BODIES=spmv,spmvvec timeout 600 python tools/chunk_trace.py 1:1:0,1:1:1:1,2:1:0 > gpurun_out/r02ab/trace.jsonl 2> gpurun_out/r02ab/trace.err
cat gpurun_out/r02ab/trace.jsonl; tail -3 gpurun_out/r02ab/trace.err
