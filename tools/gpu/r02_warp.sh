#!/bin/bash
# R30 warp-task worker: GPU tests, then the (C, prefetch, warp) sweep of the configs[1] kernels.
mkdir -p gpurun_out/r02w
timeout 900 python -m pytest tests/test_gpu_warp_tasks.py -x -q > gpurun_out/r02w/pytest_warp.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/r02w/pytest_warp.log
timeout 600 python tools/sweep_ck.py --bodies spmvvec,spmv,stencil --chunks 1,2,4,8,16 --prefetch 0,1 --warp 0,1 --reps 20 > gpurun_out/r02w/sweep.jsonl 2> gpurun_out/r02w/sweep.err; echo "sweep rc=$?"
cat gpurun_out/r02w/sweep.jsonl
