#!/bin/bash
# licence slack A/B for the in-tile CTA-pair GEMM: throughput (gemm_perf) and drain latency
mkdir -p gpurun_out/r02g2
for v in lic0 default lic4; do
  if [ $v = default ]; then unset FLEP_LIB_PATH; else export FLEP_LIB_PATH=$PWD/build_variants/$v.so; fi
  timeout 300 python tools/gemm_perf.py > gpurun_out/r02g2/perf_$v.jsonl 2>&1
  timeout 300 python bench.py --config gemm --gemm-pair 1 --gemm-in-tile 1 --steps 30 --warmup 3 \
    > gpurun_out/r02g2/lat_$v.json 2>&1
  echo "$v $(grep -h gemm2_flep gpurun_out/r02g2/perf_$v.jsonl | cut -c30-110 | tr '\n' ' ')"
  echo "$v $(grep -o '"drain_us": {[^}]*}' gpurun_out/r02g2/lat_$v.json) bad=$(grep -o '"not_bit_identical_to_uninterrupted": [0-9]*' gpurun_out/r02g2/lat_$v.json)"
done
unset FLEP_LIB_PATH
timeout 600 python -m pytest tests/test_gpu_gemm2.py -x -q 2>&1 | tail -2
