#!/bin/bash
# queues (configs[3], configs[4] N=1) with the in-tile 1-CTA GEMM (1) vs the in-tile CTA-pair GEMM (2)
mkdir -p gpurun_out/r02qg2
for g in 1 2 1 2; do
  FLEP_QUEUE_GEMM=$g timeout 300 python bench.py --config queue > gpurun_out/r02qg2/q$g.json 2>gpurun_out/r02qg2/q$g.err
  FLEP_QUEUE_GEMM=$g timeout 300 python bench.py --config scale > gpurun_out/r02qg2/s$g.json 2>gpurun_out/r02qg2/s$g.err
  cat gpurun_out/r02qg2/q$g.json >> gpurun_out/r02qg2/q_all.jsonl
  cat gpurun_out/r02qg2/s$g.json >> gpurun_out/r02qg2/s_all.jsonl
  python -c "
import json
q=json.loads(open('gpurun_out/r02qg2/q$g.json').read().strip().splitlines()[-1])
print('queue gemm$g', q['antt'], q['makespan_ms'], {k:v for k,v in q['t_alone_us'].items() if 'gemm' in k})
s=json.loads(open('gpurun_out/r02qg2/s$g.json').read().strip().splitlines()[-1])
print('scale gemm$g', s.get('value'), s.get('unit'), {k: s[k] for k in s if 'latency' in k or 'antt' in k})"
done
