#!/bin/bash
# Round 2: the managed spatial config alone, then the default bench line with the
# configs[0,2,3,4] sub-records (as the driver runs it); evidence logs under gpurun_out/r02.
mkdir -p gpurun_out/r02
export FLEP_EVIDENCE_DIR=gpurun_out/r02
timeout 300 python bench.py --config spatial_managed --steps 6 --warmup 3 > gpurun_out/r02/spatial_managed.json 2> gpurun_out/r02/spatial_managed.err; echo "spatial_managed rc=$?"
tail -c 1500 gpurun_out/r02/spatial_managed.err
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r02/bench_full.json 2> gpurun_out/r02/bench_full.err; echo "bench rc=$?"
tail -c 1500 gpurun_out/r02/bench_full.err
python - <<'PY'
import json
d = json.loads(open("gpurun_out/r02/bench_full.json").read().strip().splitlines()[-1])
print("value", d["value"], "wall", d.get("configs", {}).get("wall_s"))
for k, v in d.get("configs", {}).items():
    if isinstance(v, dict) and "value" in v:
        print(k, v["value"], v.get("unit"))
PY
