#!/bin/bash
# SpMV in-flight gathers per thread (FLEP_SPMV_U) experiment: stencil/SpMV breakdown per build.
mkdir -p gpurun_out
for U in 4 6 8; do
  export FLEP_NVCC_EXTRA="-DFLEP_SPMV_U=$U"
  python -c "from paper_conf_asplos_wulzj17_b200 import build; build.build(force=True)"
  timeout 300 python tools/overhead_breakdown.py 1:1:0:0,2:1:0:0 2>&1 | grep spmv | sed "s/^/{\"U\": $U, \"row\": /; s/$/}/" >> gpurun_out/spmv_u.jsonl
done
