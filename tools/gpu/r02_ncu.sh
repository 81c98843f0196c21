#!/bin/bash
# ncu evidence for the round-2 bench line: the launch list of the default command (cold-cache,
# serialised: compare shares), and --set full captures of the dominant kernel (SpMV worker,
# C = K = 1) and its unwrapped twin; the probe-6 gather kernel for the limiter attribution.
mkdir -p gpurun_out/r02n
ncu --metrics gpu__time_duration.sum --clock-control none -c 800 --csv --log-file gpurun_out/r02n/launches.csv \
    python bench.py --steps 3 --warmup 3 --reps 3 --e2e-steps 2 --sub 0 > gpurun_out/r02n/bench_under_ncu.log 2>&1
echo "launch list rc=$?"
ncu --set full --clock-control none --import-source on -k regex:flep_ -c 4 -o gpurun_out/r02n/prof_full \
    python tools/profile_kernels.py --kernels spmv,stencil --reps 1 --combos 1:1:0 > gpurun_out/r02n/ncu_full.log 2>&1
echo "full rc=$?"
ncu -i gpurun_out/r02n/prof_full.ncu-rep --page raw --csv > gpurun_out/r02n/prof_full_raw.csv 2>&1
ncu -i gpurun_out/r02n/prof_full.ncu-rep --page details --csv > gpurun_out/r02n/prof_full_details.csv 2>&1
