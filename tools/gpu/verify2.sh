#!/bin/bash
# GPU parity suite + default bench line + amortizing-factor tuning table
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
[ -n "$NO_BENCH" ] && exit 0
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo "bench rc=$?"
timeout 900 python bench.py --config tune > gpurun_out/bench_tune.json 2> gpurun_out/bench_tune.err; echo "tune rc=$?"
