#!/bin/bash
# wide pair GEMM: tests, preemption latency (bench --config gemm, pair = 1 / 2, in-tile), and the
# configs[3] / configs[4] queues with the 1-CTA (1) vs the wide pair (3) GEMM body
mkdir -p gpurun_out/r02wq
timeout 900 python -m pytest -x -q tests/test_gpu_gemm2w.py > gpurun_out/r02wq/tests.log 2>&1
rc=$?; echo "tests rc=$rc"; tail -3 gpurun_out/r02wq/tests.log
[ $rc -eq 0 ] || exit 1
for p in 1 2; do
  timeout 300 python bench.py --config gemm --gemm-pair $p --gemm-in-tile 1 --steps 30 --warmup 3 \
    > gpurun_out/r02wq/gemm_pair$p.json 2> gpurun_out/r02wq/gemm_pair$p.err
  echo "gemm pair=$p rc=$?"
done
for g in 1 3; do
  FLEP_QUEUE_GEMM=$g timeout 300 python bench.py --config queue > gpurun_out/r02wq/q$g.json 2>gpurun_out/r02wq/q$g.err; echo "queue $g rc=$?"
  FLEP_QUEUE_GEMM=$g timeout 300 python bench.py --config scale > gpurun_out/r02wq/s$g.json 2>gpurun_out/r02wq/s$g.err; echo "scale $g rc=$?"
done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/r02wq/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "ERR", e); continue
    keep = {k: d.get(k) for k in ("value", "unit", "drain_us", "not_bit_identical_to_uninterrupted", "antt", "natt_gain_vs_fifo", "throughput_kernels_per_s", "preemption_latency_us")}
    print(f, json.dumps(keep)[:600])
PY
