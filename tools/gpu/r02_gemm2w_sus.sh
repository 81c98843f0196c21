#!/bin/bash
# sustained (power-capped) 8192^3 comparison: cuBLAS, 256x256 pair, 256x512 pair; energy per GEMM
mkdir -p gpurun_out/r02w
GEMM_SUSTAINED_S=${GEMM_SUSTAINED_S:-2} GEMM_ROUNDS=${GEMM_ROUNDS:-2} \
GEMM_ONLY=${GEMM_ONLY:-gemm2_static_u1,gemm2_flep_c1,gemm2w_static_u1,gemm2w_flep_c1,gemm2w_flep_c1_intile,gemm2_flep_c1_intile} \
  timeout 900 python tools/gemm_perf.py > gpurun_out/r02w/gemm_sustained.jsonl 2> gpurun_out/r02w/gemm_sustained.err
echo "rc=$?"; cat gpurun_out/r02w/gemm_sustained.jsonl; tail -3 gpurun_out/r02w/gemm_sustained.err
