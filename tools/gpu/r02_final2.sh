#!/bin/bash
# Final evidence with the speculative-fetch victim (R34): smoke, default bench line, reference arm,
# the ncu launch list of the bench command and --set full of the dominant kernel (SpMV worker with
# R34, C = K = 1) and its unwrapped twin; compute-sanitizer over the sanitizer case.
mkdir -p gpurun_out/r02g
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/r02g/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/r02g/smoke.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r02g/bench.json 2> gpurun_out/r02g/bench.err; echo "bench rc=$?"
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/r02g/ref.json 2> gpurun_out/r02g/ref.err; echo "ref rc=$?"
ncu --metrics gpu__time_duration.sum --clock-control none -c 800 --csv --log-file gpurun_out/r02g/launches.csv \
    python bench.py --steps 3 --warmup 3 --reps 3 --e2e-steps 2 --sub 0 > gpurun_out/r02g/bench_under_ncu.log 2>&1
echo "launch list rc=$?"
ncu --set full --clock-control none --import-source on -k regex:flep_ -c 4 -o gpurun_out/r02g/prof_full \
    python tools/profile_kernels.py --kernels spmv --reps 1 --combos 1:1:0:0:0:1,1:1:0 > gpurun_out/r02g/ncu_full.log 2>&1
echo "full rc=$?"
ncu -i gpurun_out/r02g/prof_full.ncu-rep --page raw --csv > gpurun_out/r02g/prof_full_raw.csv 2>&1
for tool in memcheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --target-processes all python tools/sanitizer_case.py > gpurun_out/r02g/sanitizer_$tool.log 2>&1
  echo "$tool rc=$? $(tail -1 gpurun_out/r02g/sanitizer_$tool.log)"
done
python - <<'PY'
import json
d = json.loads(open("gpurun_out/r02g/bench.json").read().strip().splitlines()[-1])
print("value", d["value"], "e2e", d["e2e"]["value"], "frac", d["roofline"]["frac"], "clocks", d["clocks"])
print({k: v.get("overhead_pct") for k, v in d["kernels"].items() if isinstance(v, dict)})
r = json.loads(open("gpurun_out/r02g/ref.json").read().strip().splitlines()[-1])
print("ref", r["value"], r["ms_per_step"])
PY
