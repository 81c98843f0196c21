#!/bin/bash
# scheduler state in shared memory vs registers (-DFLEP_SCHED_IN_REGS): GPU tests, then an
# interleaved A/B of the configs[1] kernels' workers, two rounds
mkdir -p gpurun_out/r02ss
timeout 1500 python -m pytest -x -q tests/test_gpu_spec_fetch.py tests/test_gpu_parity.py tests/test_gpu_runtime.py > gpurun_out/r02ss/tests.log 2>&1
rc=$?; echo "tests rc=$rc"; tail -3 gpurun_out/r02ss/tests.log
[ $rc -eq 0 ] || exit 1
CASES=spmv:1:1:0:0:0:0:0:0:1,spmv:2:1:0:0:0:0:0:0:1,spmv:1:1,spmvvec:1:1,stencil:1:1:0:0:0:0:0:0:1,stencil:2:1
for rep in 1 2; do
for v in smem regs; do
  FLEP_LIB_PATH=build_variants/$v.so timeout 300 python tools/ab_overhead.py $CASES >> gpurun_out/r02ss/ab.jsonl 2>> gpurun_out/r02ss/ab.err
done
done
python - <<'PY'
import json
for l in open("gpurun_out/r02ss/ab.jsonl"):
    if l.startswith("{"):
        d = json.loads(l); print(d["lib"], d["case"], d["wrapped_us"], d["unwrapped_us"], d["overhead_pct"])
PY
tail -2 gpurun_out/r02ss/ab.err
