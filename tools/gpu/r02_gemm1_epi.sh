#!/bin/bash
# 1-CTA GEMM with the bulk-store epilogue: parity tests (1-CTA and pair), 8192^3 timing, in-tile
# drain, and the queues that use the 1-CTA body
mkdir -p gpurun_out/r02g1
timeout 1200 python -m pytest -x -q tests/test_gpu_gemm.py tests/test_gpu_gemm2.py tests/test_gpu_gemm2w.py > gpurun_out/r02g1/tests.log 2>&1
rc=$?; echo "tests rc=$rc"; tail -3 gpurun_out/r02g1/tests.log
[ $rc -eq 0 ] || exit 1
GEMM_REPS=16 GEMM_ONLY=gemm1_unwrapped,gemm1_static_u1,gemm1_flep_c1,gemm1_flep_c2_intile,gemm2w_flep_c1 timeout 600 python tools/gemm_perf.py > gpurun_out/r02g1/perf.jsonl 2> gpurun_out/r02g1/perf.err
cut -c1-150 gpurun_out/r02g1/perf.jsonl
GEMM_SUSTAINED_S=2 GEMM_ROUNDS=1 GEMM_ONLY=gemm1_flep_c1,gemm1_flep_c2_intile,gemm2w_flep_c1 timeout 600 python tools/gemm_perf.py > gpurun_out/r02g1/sus.jsonl 2> gpurun_out/r02g1/sus.err
cut -c1-220 gpurun_out/r02g1/sus.jsonl
timeout 300 python bench.py --config gemm --gemm-pair 0 --gemm-in-tile 1 --steps 30 --warmup 3 > gpurun_out/r02g1/gemm_preempt.json 2> gpurun_out/r02g1/gemm_preempt.err
python -c "import json; d=json.loads(open('gpurun_out/r02g1/gemm_preempt.json').read().strip().splitlines()[-1]); print('drain', d['drain_us'], 'bad', d['not_bit_identical_to_uninterrupted'])"
timeout 300 python bench.py --config queue > gpurun_out/r02g1/q.json 2>gpurun_out/r02g1/q.err; echo "queue rc=$?"
timeout 300 python bench.py --config scale > gpurun_out/r02g1/s.json 2>gpurun_out/r02g1/s.err; echo "scale rc=$?"
python -c "
import json
d=json.loads(open('gpurun_out/r02g1/q.json').read().strip().splitlines()[-1]); print('q', d['value'], d['antt'], d['t_alone_us'])
d=json.loads(open('gpurun_out/r02g1/s.json').read().strip().splitlines()[-1]); print('s', d['value'], d['preempt_latency_us_all'], d['aggregate']['HPF'])"
