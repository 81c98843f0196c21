#!/bin/bash
# wide CTA-pair GEMM (256x512 tiles): parity tests, then the 8192^3 interleaved timing
mkdir -p gpurun_out/r02w
timeout 900 python -m pytest -x -q tests/test_gpu_gemm2w.py tests/test_gpu_gemm2.py > gpurun_out/r02w/tests.log 2>&1
echo "tests rc=$?"; tail -5 gpurun_out/r02w/tests.log
GEMM_ONLY=${GEMM_ONLY:-gemm2_unwrapped,gemm2_static_u1,gemm2_flep_c2,gemm2w_unwrapped,gemm2w_static_u1,gemm2w_flep_c1,gemm2w_flep_c2,gemm2w_flep_c1_intile} \
  GEMM_REPS=${GEMM_REPS:-24} timeout 600 python tools/gemm_perf.py > gpurun_out/r02w/gemm_perf.jsonl 2> gpurun_out/r02w/gemm_perf.err
echo "perf rc=$?"; cut -c1-170 gpurun_out/r02w/gemm_perf.jsonl; tail -3 gpurun_out/r02w/gemm_perf.err
