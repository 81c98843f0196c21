#!/bin/bash
mkdir -p gpurun_out/r02t
export FLEP_EVIDENCE_DIR=gpurun_out/r02t
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r02t/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -25 gpurun_out/r02t/pytest_gpu.log
