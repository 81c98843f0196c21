#!/bin/bash
# One gpurun call: GPU parity suite, default bench line, exit-accounting probe.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/probe4 probes/probe4.cu && /tmp/probe4 > gpurun_out/probe4.jsonl 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo "bench rc=$?"
tail -3 gpurun_out/pytest_gpu.log
