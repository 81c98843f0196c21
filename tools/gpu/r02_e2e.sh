#!/bin/bash
# e2e (managed HPF, host buffers) with and without the speculative fetch, 40 steps each, twice
mkdir -p gpurun_out/r02e
for r in 1 2; do for sp in 1 0; do
  timeout 600 python bench.py --steps 5 --warmup 3 --e2e-steps 40 --sub 0 --op2 0 --lp-spec $sp > gpurun_out/r02e/e2e_${sp}_$r.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/r02e/e2e_${sp}_$r.json').read().strip().splitlines()[-1]); e=d['e2e']
print('spec=$sp run=$r', 'value', d['value'], 'e2e', e['value'], e['breakdown_us_p50'], e['host_path_us_p50'])"
done; done
