#!/bin/bash
mkdir -p gpurun_out/r02ab
for v in build_variants/*.so; do
  FLEP_LIB_PATH=$v timeout 300 python tools/ab_overhead.py "$@" >> gpurun_out/r02ab/ab.jsonl 2>> gpurun_out/r02ab/ab.err
done
cat gpurun_out/r02ab/ab.jsonl; tail -3 gpurun_out/r02ab/ab.err
