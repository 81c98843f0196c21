#!/bin/bash
# ncu --set full: cuBLAS beside the 256x256 and the 256x512 pair bodies (static twins, TMA-store
# epilogue) at 8192^3
mkdir -p gpurun_out/r02gn2
export GEMM_ONLY=gemm2_static_u1,gemm2w_static_u1,gemm2w_flep_c1 GEMM_REPS=1
timeout 300 python tools/gemm_perf.py > gpurun_out/r02gn2/plain.jsonl 2> gpurun_out/r02gn2/plain.err && \
ncu --set full --clock-control none --import-source on -k regex:'flep_gemm2|nvjet|cutlass|sm100|gemm' -c 4 \
    -o gpurun_out/r02gn2/gemm python tools/gemm_perf.py > gpurun_out/r02gn2/ncu.log 2>&1
echo "ncu rc=$?"
ncu -i gpurun_out/r02gn2/gemm.ncu-rep --page raw --csv > gpurun_out/r02gn2/raw.csv 2>&1
python tools/ncu_gemm_summary.py gpurun_out/r02gn2/raw.csv > gpurun_out/r02gn2/summary.json
grep -c kernel gpurun_out/r02gn2/summary.json
