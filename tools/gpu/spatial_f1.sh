#!/bin/bash
# Measure this box's smid -> die map (probe 7), then the spatial f1 experiments with it.
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/probe7 probes/probe7.cu && /tmp/probe7 > gpurun_out/probe7_box.json
python - <<'PY'
import json, numpy as np
d = json.load(open("gpurun_out/probe7_box.json"))
M = np.array(d["matrix"]); X = M - M.mean(axis=1, keepdims=True); X = X - X.mean(axis=0, keepdims=True)
u, s, vt = np.linalg.svd(X, full_matrices=False)
die = (vt[0] > np.median(vt[0])).astype(int)
if die[0] == 1: die = 1 - die
json.dump({"die": [int(x) for x in die], "singular_values": [float(x) for x in s[:3]]}, open("gpurun_out/die_map_box.json", "w"))
PY
timeout 300 python -m pytest tests/test_gpu_runtime.py -k rank_table -q 2>&1 | tail -1
FLEP_DIE_MAP=gpurun_out/die_map_box.json timeout 1500 python bench.py --config spatial_f1 --steps 80 > gpurun_out/spatial_f1.json 2> gpurun_out/spatial_f1.err; echo "rc=$?"
