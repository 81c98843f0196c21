#!/bin/bash
# cp.async SpMV body experiment (FLEP_SPMV_ASYNC=1) at AU = 4, 8: SpMV parity tests, overhead sweep, bench.
mkdir -p gpurun_out
for AU in 8 4; do
  export FLEP_NVCC_EXTRA="-DFLEP_SPMV_ASYNC=1 -DFLEP_SPMV_AU=$AU"
  python -c "from paper_conf_asplos_wulzj17_b200 import build; build.build(force=True)"
  timeout 600 python -m pytest tests -m gpu -q -x -k "spmv or smoke or schedules" > gpurun_out/async_tests_$AU.log 2>&1; echo "rc=$?" >> gpurun_out/async_tests_$AU.log
  timeout 300 python tools/sweep_ck.py --bodies spmv --chunks 1,2 --prefetch 0 --reps 20 > gpurun_out/async_sweep_$AU.jsonl 2>&1
  timeout 300 python bench.py --steps 100 --warmup 5 --e2e-steps 3 > gpurun_out/async_bench_$AU.json 2> gpurun_out/async_bench_$AU.err
done
