#!/bin/bash
# CSR-vector SpMV body experiment (FLEP_SPMV_VECTOR=1) at U = 2, 4: parity tests + timings.
mkdir -p gpurun_out; rm -f gpurun_out/spmv_vec.jsonl
for U in 2 4; do
  export FLEP_NVCC_EXTRA="-DFLEP_SPMV_VECTOR=1 -DFLEP_SPMV_U=$U"
  python -c "from paper_conf_asplos_wulzj17_b200 import build; build.build(force=True)"
  timeout 600 python -m pytest tests -m gpu -q -k "spmv" 2>&1 | tail -1
  timeout 300 python tools/overhead_breakdown.py 1:1:0:0,2:1:0:0 2>&1 | grep spmv | sed "s/^/{\"U\": $U, \"row\": /; s/$/}/" >> gpurun_out/spmv_vec.jsonl
done
