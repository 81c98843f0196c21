#!/bin/bash
# functional run of the N = 2 path on one GPU (two ranks share it; gloo process group)
mkdir -p gpurun_out/r02n2
FLEP_SHARE_GPU=1 timeout 900 python bench.py --gpus 2 --steps 5 --warmup 3 --reps 8 --e2e-steps 3 > gpurun_out/r02n2/bench_n2.json 2> gpurun_out/r02n2/bench_n2.err; echo "n2 rc=$?"
tail -c 2000 gpurun_out/r02n2/bench_n2.err | grep -v Warning | tail -20
python - <<'PY'
import json
lines = [l for l in open("gpurun_out/r02n2/bench_n2.json").read().splitlines() if l.startswith("{")]
print("json lines:", len(lines))
d = json.loads(lines[-1])
print("n_gpus", d["n_gpus"], "value", d["value"], "c4", d["configs"]["configs[4]"]["value"], [g["kernels"] for g in d["configs"]["configs[4]"]["per_gpu"]])
PY
