#!/bin/bash
# wide/narrow pair GEMM after a change: parity tests, interleaved timing, sustained timing + energy
mkdir -p gpurun_out/r02w
timeout 900 python -m pytest -x -q tests/test_gpu_gemm2w.py tests/test_gpu_gemm2.py > gpurun_out/r02w/tests.log 2>&1
rc=$?; echo "tests rc=$rc"; tail -5 gpurun_out/r02w/tests.log
[ $rc -eq 0 ] || exit 1
GEMM_REPS=24 GEMM_ONLY=gemm2_unwrapped,gemm2_static_u1,gemm2_flep_c1,gemm2_flep_c2,gemm2w_unwrapped,gemm2w_static_u1,gemm2w_flep_c1,gemm2w_flep_c1_intile \
  timeout 600 python tools/gemm_perf.py > gpurun_out/r02w/gemm_perf.jsonl 2> gpurun_out/r02w/gemm_perf.err
echo "perf rc=$?"; cut -c1-130 gpurun_out/r02w/gemm_perf.jsonl
tools/gpu/r02_gemm2w_sus.sh | cut -c1-220
