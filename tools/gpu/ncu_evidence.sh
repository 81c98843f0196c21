#!/bin/bash
# ncu evidence for the bench line: launch list of the bench command, and --set full captures of the
# wrapped / unwrapped SpMV and stencil kernels (the bench's dominant kernel is the SpMV worker).
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 3 --warmup 3 --reps 3 --e2e-steps 2 > gpurun_out/bench_under_ncu.log 2>&1
echo "launch list rc=$?"
ncu --set full --clock-control none --import-source on -k regex:flep_ -c 4 -o gpurun_out/prof_full \
    python tools/profile_kernels.py --kernels spmv,stencil --reps 1 --combos 1:1:0 > gpurun_out/ncu_full.log 2>&1
echo "full rc=$?"
ncu -i gpurun_out/prof_full.ncu-rep --page raw --csv > gpurun_out/prof_full_raw.csv 2>&1
