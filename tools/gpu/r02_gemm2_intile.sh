#!/bin/bash
# in-tile preemption of the CTA-pair GEMM: throughput beside cuBLAS and the other forms, the
# full-GPU preemption latency of the pair victim (in-tile and tile granularity), sanitizers
mkdir -p gpurun_out/r02g2
timeout 300 python tools/gemm_perf.py > gpurun_out/r02g2/gemm_perf.jsonl 2> gpurun_out/r02g2/gemm_perf.err
for it in 1 0; do
  timeout 300 python bench.py --config gemm --gemm-pair 1 --gemm-in-tile $it --steps 30 --warmup 3 \
    > gpurun_out/r02g2/gemm_pair_intile$it.json 2> gpurun_out/r02g2/gemm_pair_intile$it.err
done
timeout 300 python bench.py --config gemm --gemm-pair 0 --gemm-in-tile 1 --steps 30 --warmup 3 \
  > gpurun_out/r02g2/gemm_1cta_intile1.json 2> gpurun_out/r02g2/gemm_1cta_intile1.err
for tool in memcheck synccheck racecheck; do
  timeout 900 compute-sanitizer --tool $tool --target-processes all python tools/sanitizer_case.py > gpurun_out/r02g2/sanitizer_$tool.log 2>&1
  echo "$tool rc=$? $(tail -1 gpurun_out/r02g2/sanitizer_$tool.log)"
done
tail -c 600 gpurun_out/r02g2/*.json*
