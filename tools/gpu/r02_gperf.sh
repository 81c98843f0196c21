#!/bin/bash
mkdir -p gpurun_out/r02g
timeout 600 python tools/gemm_perf.py > gpurun_out/r02g/gemm_perf.jsonl 2> gpurun_out/r02g/gemm_perf.err; echo "rc=$?"
cut -c1-200 gpurun_out/r02g/gemm_perf.jsonl; tail -3 gpurun_out/r02g/gemm_perf.err
