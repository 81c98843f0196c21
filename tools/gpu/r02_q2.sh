#!/bin/bash
mkdir -p gpurun_out/r02q2
export FLEP_EVIDENCE_DIR=gpurun_out/r02q2
FLEP_DEBUG_SLOW=300 timeout 600 python bench.py --config queue > gpurun_out/r02q2/queue.json 2> gpurun_out/r02q2/queue.err; echo "queue rc=$?"
grep -c "flep" gpurun_out/r02q2/queue.err; grep "flep" gpurun_out/r02q2/queue.err | head -30
nproc; uptime
