#!/bin/bash
# Round 2, first GPU call: the GPU parity suite on the new build, the default bench line, the
# random-gather ceiling attribution (ncu --set full of probe 6's best case), the L2-persisting
# window probe (probe 9).
mkdir -p gpurun_out/r02
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r02/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02/pytest_gpu.log
tail -3 gpurun_out/r02/pytest_gpu.log
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/r02/bench_default.json 2> gpurun_out/r02/bench_default.err; echo "bench rc=$?"
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o /tmp/probe6 probes/probe6.cu && /tmp/probe6 > gpurun_out/r02/probe6.jsonl
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o /tmp/probe9 probes/probe9.cu && /tmp/probe9 > gpurun_out/r02/probe9.jsonl
timeout 300 ncu --set full --clock-control none -k regex:k_gather -s 110 -c 1 -o gpurun_out/r02/probe6_full /tmp/probe6 > gpurun_out/r02/probe6_ncu.log 2>&1
ncu -i gpurun_out/r02/probe6_full.ncu-rep --page raw --csv > gpurun_out/r02/probe6_full_raw.csv 2>&1
echo done
