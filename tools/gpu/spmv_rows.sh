#!/bin/bash
# SpMV original-block size experiment: build with FLEP_SPMV_ROWS=R, run the default bench line.
mkdir -p gpurun_out
for R in 64 32; do
  export FLEP_NVCC_EXTRA="-DFLEP_SPMV_ROWS=$R" FLEP_SPMV_ROWS=$R
  python -c "from paper_conf_asplos_wulzj17_b200 import build; build.build(force=True)"
  timeout 600 python bench.py --steps 100 > gpurun_out/bench_rows$R.json 2> gpurun_out/bench_rows$R.err; echo "rows $R rc=$?"
done
