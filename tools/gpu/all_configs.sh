#!/bin/bash
# Every bench configuration once (round-end evidence refresh); one JSON line per file.
mkdir -p gpurun_out/cfg
for c in corun1 spatial gemm ffs model clc delay; do
  timeout 900 python bench.py --config $c > gpurun_out/cfg/$c.json 2> gpurun_out/cfg/$c.err
  echo "$c rc=$?"
done
timeout 300 python bench.py --impl reference > gpurun_out/cfg/reference.json 2> gpurun_out/cfg/reference.err; echo "reference rc=$?"
