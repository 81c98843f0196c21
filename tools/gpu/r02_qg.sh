#!/bin/bash
mkdir -p gpurun_out/r02qg
timeout 600 python -m pytest tests/test_gpu_gemm2.py -x -q > gpurun_out/r02qg/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r02qg/pytest.log
for g in 1 2 1 2; do
  FLEP_QUEUE_GEMM=$g timeout 300 python bench.py --config queue > gpurun_out/r02qg/q$g.json 2>gpurun_out/r02qg/q$g.err
  python -c "
import json; q=json.loads(open('gpurun_out/r02qg/q$g.json').read().strip().splitlines()[-1])
print('gemm$g', q['antt'], q['makespan_ms'], {k:v for k,v in q['t_alone_us'].items() if 'gemm' in k})"
done
