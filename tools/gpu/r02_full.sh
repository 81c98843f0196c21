#!/bin/bash
# the default bench line as the driver runs it, then the GPU suite
mkdir -p gpurun_out/r02f
export FLEP_EVIDENCE_DIR=gpurun_out/r02f
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r02f/bench.json 2> gpurun_out/r02f/bench.err; echo "bench rc=$?"


