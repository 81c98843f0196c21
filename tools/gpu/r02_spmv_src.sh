#!/bin/bash
# source-level stall attribution of the bench victim (SpMV counter worker, C = K = 1, speculative
# fetch) and its unwrapped twin: which instructions the warps wait on
mkdir -p gpurun_out/r02src
timeout 300 python tools/profile_kernels.py --kernels spmv --reps 1 --combos 1:1:0:0:0:1 > gpurun_out/r02src/plain.log 2>&1 && \
ncu --set full --clock-control none --import-source on -k regex:flep_ -c 2 -o gpurun_out/r02src/prof \
    python tools/profile_kernels.py --kernels spmv --reps 1 --combos 1:1:0:0:0:1 > gpurun_out/r02src/ncu.log 2>&1
echo "ncu rc=$?"
ncu -i gpurun_out/r02src/prof.ncu-rep --page source --csv --print-source sass > gpurun_out/r02src/source_sass.csv 2>&1
ncu -i gpurun_out/r02src/prof.ncu-rep --page source --csv > gpurun_out/r02src/source.csv 2>&1
ncu -i gpurun_out/r02src/prof.ncu-rep --page raw --csv > gpurun_out/r02src/raw.csv 2>&1
ls -la gpurun_out/r02src; head -c 600 gpurun_out/r02src/source.csv
