#!/bin/bash
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_relay.py -q -x > gpurun_out/pytest_relay.log 2>&1; rc=$?; tail -1 gpurun_out/pytest_relay.log
[ $rc -ne 0 ] && exit 1
for R in 0 1; do for O in 0 1; do
  timeout 240 python bench.py --steps 10 --e2e-steps 40 --e2e-relay $R --e2e-overlap-copy $O > gpurun_out/e2e_r${R}_o${O}.json 2>/dev/null
done; done
