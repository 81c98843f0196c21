#!/bin/bash
mkdir -p gpurun_out/r02
timeout 600 python -m pytest tests/test_gpu_runtime.py -x -q -k "spatial_hpf or managed_cancel or managed_hpf or cancel" > gpurun_out/r02/pytest_rt.log 2>&1; echo "pytest rc=$?"; tail -30 gpurun_out/r02/pytest_rt.log
