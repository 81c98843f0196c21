#!/bin/bash
mkdir -p gpurun_out/r02
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r02/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -25 gpurun_out/r02/pytest_gpu.log
