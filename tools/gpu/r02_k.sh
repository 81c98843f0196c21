#!/bin/bash
mkdir -p gpurun_out/r02k
FLEP_LIB_PATH= timeout 300 python tools/ab_overhead.py spmv:1:1,spmv:1:1000,spmv:2:1,spmv:2:1000,spmvvec:1:1,spmvvec:1:1000,stencil:1:1,stencil:1:1000,stencil:1:1:0:1,stencil:1:1000:0:1,spmv:1:1:0:1,spmv:1:1000:0:1 > gpurun_out/r02k/ab.jsonl 2> gpurun_out/r02k/ab.err
cut -c1-220 gpurun_out/r02k/ab.jsonl; tail -3 gpurun_out/r02k/ab.err
