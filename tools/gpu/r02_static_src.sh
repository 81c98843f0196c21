#!/bin/bash
# ncu source view: the static-schedule worker (R37, async poll) vs the static twin, stencil 4096^2
mkdir -p gpurun_out/r02ssrc
ARGS="--kernels stencil --reps 1 --combos 1:1:0:1:0:0:1 --static-twin 1"
timeout 300 python tools/profile_kernels.py $ARGS > gpurun_out/r02ssrc/plain.log 2>&1 && \
ncu --set full --clock-control none --import-source on -k regex:'flep_worker_static|flep_static' -c 2 -o gpurun_out/r02ssrc/prof \
    python tools/profile_kernels.py $ARGS > gpurun_out/r02ssrc/ncu.log 2>&1
echo "ncu rc=$?"
ncu -i gpurun_out/r02ssrc/prof.ncu-rep --page source --csv > gpurun_out/r02ssrc/source.csv 2>&1
ncu -i gpurun_out/r02ssrc/prof.ncu-rep --page raw --csv > gpurun_out/r02ssrc/raw.csv 2>&1
ls -la gpurun_out/r02ssrc | head
