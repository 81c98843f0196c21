#!/bin/bash
# queue fetch mode for the memory-bound bodies: prefetch (A4: the held chunk runs before a yield)
# vs speculative fetch (R34: the held chunk goes back through the record); configs[3] and [4]
mkdir -p gpurun_out/r02qs
for rep in 1 2; do
for m in prefetch spec; do
  FLEP_QUEUE_FETCH=$m timeout 300 python bench.py --config queue > gpurun_out/r02qs/q_${m}_$rep.json 2>gpurun_out/r02qs/q_${m}_$rep.err; echo "queue $m rc=$?"
  FLEP_QUEUE_FETCH=$m timeout 300 python bench.py --config scale > gpurun_out/r02qs/s_${m}_$rep.json 2>gpurun_out/r02qs/s_${m}_$rep.err; echo "scale $m rc=$?"
done
done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/r02qs/*.json")):
    d = json.loads(open(f).read().strip().splitlines()[-1])
    if "antt" in d:
        print(f, "NATT", d.get("value"), "ANTT HPF", d["antt"].get("HPF"), "FIFO", d["antt"].get("FIFO"), "makespan HPF", d["makespan_ms"].get("HPF"))
    else:
        print(f, "NATT", d["value"], "lat", d["preempt_latency_us_all"], "thr", d["aggregate"]["HPF"]["throughput_kernels_per_s"])
        print("   ", json.dumps(d["preempt_latency_us_by_victim"]))
        print("   ", json.dumps(d["wrapper_overhead_pct_rank0"]))
PY
