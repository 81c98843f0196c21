#!/bin/bash
# Every bench configuration once on the final build (evidence refresh); one JSON line per file.
mkdir -p gpurun_out/cfgf
for c in corun1 spatial spatial_managed spatial_f1 queue scale slicing coruns gemm ffs model tune clc delay; do
  s=$(date +%s)
  timeout 900 python bench.py --config $c > gpurun_out/cfgf/$c.json 2> gpurun_out/cfgf/$c.err
  echo "$c rc=$? $(( $(date +%s) - s ))s"
done
timeout 600 python bench.py --config gemm --gemm-pair 2 > gpurun_out/cfgf/gemm_wide.json 2> gpurun_out/cfgf/gemm_wide.err; echo "gemm wide rc=$?"
