"""The N > 1 bench path on a real GPU: `bench.py --gpus 2` launches two ranks
itself; with FLEP_SHARE_GPU=1 both share the box's GPU on a gloo process group (NCCL refuses a
shared GPU). Checked: exactly one JSON line, n_gpus = 2, the configs[4] sub-record partitions the
512-kernel queue over both ranks and reports both GPUs. Timing values of such a run are not
scaling measurements."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_bench_two_ranks_one_line():
    env = dict(os.environ)
    for k in ("RANK", "WORLD_SIZE", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT"):
        env.pop(k, None)
    env["FLEP_SHARE_GPU"] = "1"
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "3", "--warmup", "3",
                        "--reps", "4", "--e2e-steps", "2", "--sub-steps", "3",
                        "--skip-sub", "configs[2],configs[2]_managed,configs[3],E13_never_preempted,coruns_E4_E6_E8"],
                       capture_output=True, text=True, env=env, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2
    c4 = d["configs"]["configs[4]"]
    assert [g["rank"] for g in c4["per_gpu"]] == [0, 1]
    assert sum(g["kernels"] for g in c4["per_gpu"]) == 512
    assert d["configs"]["configs[0]"]["wrong_results"] == 0
