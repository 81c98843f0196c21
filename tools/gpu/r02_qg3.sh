#!/bin/bash
# queue GEMM body choice after R35 (bulk-store epilogue): 1-CTA in-tile (1) vs 256x256 pair in-tile (2), two runs each
mkdir -p gpurun_out/r02qg3
for rep in 1 2; do
for g in 1 2; do
  FLEP_QUEUE_GEMM=$g timeout 300 python bench.py --config queue > gpurun_out/r02qg3/q${g}_$rep.json 2>gpurun_out/r02qg3/q${g}_$rep.err; echo "queue $g rc=$?"
  FLEP_QUEUE_GEMM=$g timeout 300 python bench.py --config scale > gpurun_out/r02qg3/s${g}_$rep.json 2>gpurun_out/r02qg3/s${g}_$rep.err; echo "scale $g rc=$?"
done
done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/r02qg3/*.json")):
    d = json.loads(open(f).read().strip().splitlines()[-1])
    if "antt" in d:
        print(f, "NATT", d.get("value"), "ANTT", d.get("antt"), "makespan", d.get("makespan_ms"))
    else:
        keys = [k for k in d if "latency" in k or "throughput" in k or k in ("value",)]
        print(f, {k: d[k] for k in keys})
PY
