#!/bin/bash
# which part of the pair's in-tile path costs throughput: licence, in-tile poll or epilogue peek
mkdir -p gpurun_out/r02g2
export GEMM_ONLY=gemm2_static_u1,gemm2_flep_c1,gemm2_flep_c1_intile GEMM_REPS=20
for v in default NO_LIC NO_POLL NO_PEEK default; do
  if [ $v = default ]; then unset FLEP_LIB_PATH; else export FLEP_LIB_PATH=$PWD/build_variants/$v.so; fi
  timeout 300 python tools/gemm_perf.py > gpurun_out/r02g2/ab_$v.jsonl 2>&1
  echo "$v: $(grep -h gemm2_ gpurun_out/r02g2/ab_$v.jsonl | cut -c30-100 | tr '\n' ' ')"
done
