#!/bin/bash
mkdir -p gpurun_out/r02g
timeout 600 python -m pytest tests/test_gpu_gemm2.py -x -q > gpurun_out/r02g/pytest.log 2>&1; echo "pytest rc=$?"; tail -30 gpurun_out/r02g/pytest.log
