#!/bin/bash
mkdir -p gpurun_out/r02
export FLEP_EVIDENCE_DIR=gpurun_out/r02
FLEP_DEBUG_SLOW=30 timeout 300 python bench.py --config spatial_managed --steps 12 --warmup 3 > gpurun_out/r02/spatial_managed.json 2> gpurun_out/r02/spatial_managed.err; echo "spatial_managed rc=$?"
grep -c "slow epoch" gpurun_out/r02/spatial_managed.err; grep "flep" gpurun_out/r02/spatial_managed.err | head -20
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r02/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r02/pytest_gpu.log
