#!/bin/bash
mkdir -p gpurun_out/r02s
export FLEP_EVIDENCE_DIR=gpurun_out/r02s
timeout 900 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_relay.py -x -q -k "slice or relay" > gpurun_out/r02s/pytest.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/r02s/pytest.log
timeout 600 python bench.py --config slicing > gpurun_out/r02s/slicing.json 2> gpurun_out/r02s/slicing.err; echo "slicing rc=$?"; tail -c 800 gpurun_out/r02s/slicing.err
timeout 600 python bench.py --config queue > gpurun_out/r02s/queue.json 2> gpurun_out/r02s/queue.err; echo "queue rc=$?"; tail -c 800 gpurun_out/r02s/queue.err
