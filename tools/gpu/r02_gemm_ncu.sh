#!/bin/bash
# ncu --set full of the CTA-pair GEMM (static persistent twin) and cuBLAS at 8192^3: tensor-pipe
# activity, L2 throughput and DRAM bytes side by side (what limits the pair body?).
mkdir -p gpurun_out/r02gn
export GEMM_ONLY=gemm2_static_u1,gemm2_flep_c2 GEMM_REPS=1
timeout 300 python tools/gemm_perf.py > gpurun_out/r02gn/plain.jsonl 2> gpurun_out/r02gn/plain.err && \
ncu --set full --clock-control none --import-source on -k regex:'flep_gemm2|nvjet|cutlass|sm100|gemm' -c 3 \
    -o gpurun_out/r02gn/gemm python tools/gemm_perf.py > gpurun_out/r02gn/ncu.log 2>&1
echo "ncu rc=$?"
ncu -i gpurun_out/r02gn/gemm.ncu-rep --page raw --csv > gpurun_out/r02gn/raw.csv 2>&1
ncu -i gpurun_out/r02gn/gemm.ncu-rep --page details --csv > gpurun_out/r02gn/details.csv 2>&1
cut -c1-200 gpurun_out/r02gn/plain.jsonl
