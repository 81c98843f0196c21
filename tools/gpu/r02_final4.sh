#!/bin/bash
# Final evidence (late round 2): smoke, default bench line (20 steps), reference arm, the ncu
# launch list of the bench command and --set full of the dominant kernel (SpMV victim worker,
# C = K = 1, speculative fetch) beside its unwrapped twin
mkdir -p gpurun_out/r02f5
export FLEP_EVIDENCE_DIR=gpurun_out/r02f5
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02f5/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/r02f5/smoke.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r02f5/bench.json 2> gpurun_out/r02f5/bench.err; echo "bench rc=$?"
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/r02f5/ref.json 2> gpurun_out/r02f5/ref.err; echo "ref rc=$?"
ncu --metrics gpu__time_duration.sum --clock-control none -c 800 --csv --log-file gpurun_out/r02f5/launches.csv \
    python bench.py --steps 3 --warmup 3 --reps 3 --e2e-steps 2 --sub 0 > gpurun_out/r02f5/bench_under_ncu.log 2>&1
echo "launch list rc=$?"
ncu --set full --clock-control none --import-source on -k regex:flep_ -c 4 -o gpurun_out/r02f5/prof_full \
    python tools/profile_kernels.py --kernels spmv --reps 1 --combos 1:1:0:0:0:1,1:1:0 > gpurun_out/r02f5/ncu_full.log 2>&1
echo "full rc=$?"
ncu -i gpurun_out/r02f5/prof_full.ncu-rep --page raw --csv > gpurun_out/r02f5/prof_full_raw.csv 2>&1
python - <<'PY'
import json
d = json.loads(open("gpurun_out/r02f5/bench.json").read().strip().splitlines()[-1])
print("value", d["value"], "e2e", d["e2e"]["value"], "frac", d["roofline"]["frac"], "clocks", d["clocks"])
print("ovh", d["wrapper_overhead_pct"])
print("wall", d["configs"]["wall_s"])
r = json.loads(open("gpurun_out/r02f5/ref.json").read().strip().splitlines()[-1])
print("ref", r["value"], r["ms_per_step"], r.get("oracle_timings"))
PY
