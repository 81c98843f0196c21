#!/bin/bash
mkdir -p gpurun_out/r02
export FLEP_EVIDENCE_DIR=gpurun_out/r02
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r02/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r02/pytest_gpu.log
timeout 300 python bench.py --config spatial_managed --steps 12 --warmup 3 > gpurun_out/r02/spatial_managed.json 2> gpurun_out/r02/spatial_managed.err; echo "spatial_managed rc=$?"
tail -c 1500 gpurun_out/r02/spatial_managed.err
timeout 300 python bench.py --config scale > gpurun_out/r02/scale1.json 2> gpurun_out/r02/scale1.err; echo "scale rc=$?"
tail -c 1500 gpurun_out/r02/scale1.err
