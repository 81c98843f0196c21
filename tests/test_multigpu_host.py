"""Host-side logic of the N > 1 path on CPU with the gloo backend (world size 2): the one-queue
-> N-schedulers partition is identical on every rank, disjoint and complete, and the timing
reduction is a max over ranks (BASELINE configs[4]; replicas, no data-path
collective)."""
import json
import os
import socket
import subprocess
import sys

import pytest

from synth import gen

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import bench_configs
    jobs = gen.queue_trace(6, 128, 50_000)
    te = {("saxpy_f32", 0): 10_000, ("saxpy_f32", 1): 80_000, ("saxpy_f32", 2): 900_000}
    parts = bench_configs.assign_jobs(jobs, lambda j: te.get((j["type"], j["size_class"]),
                                                              20_000 * (1 + j["size_class"])), world)
    mine = [j["id"] for j in parts[rank]]
    # the max-over-ranks timing reduction used by bench.py
    t = torch.tensor([float(rank + 1), float(len(mine))], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    allparts = [None] * world
    dist.all_gather_object(allparts, mine)
    q.put((rank, [[j["id"] for j in p] for p in parts], allparts, t.tolist()))
    dist.destroy_process_group()


def test_job_queue_partition_gloo_world2():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort()
    (r0, parts0, gathered0, red0), (r1, parts1, gathered1, red1) = res
    assert parts0 == parts1                         # same partition computed on every rank
    assert gathered0[0] == parts0[0] and gathered0[1] == parts0[1]
    ids = sorted(parts0[0] + parts0[1])
    assert ids == list(range(128))                  # complete and disjoint
    assert len(parts0[0]) > 20 and len(parts0[1]) > 20
    assert red0 == red1 and red0[0] == 2.0           # max over ranks


def test_assign_jobs_single_gpu_keeps_order():
    import bench_configs
    jobs = gen.queue_trace(5, 40, 10_000)
    parts = bench_configs.assign_jobs(jobs, lambda j: 1000, 1)
    assert [j["id"] for j in parts[0]] == list(range(40))


def test_rank_tables_are_permutations_and_follow_the_die_map():
    import bench_configs as bc
    die = [0, 1, 1, 0, 0, 1, 0, 1]
    t = bc._rank_tables(8, die)
    for name, r in t.items():
        assert sorted(r) == list(range(8)), name
    # die-packed: every die-0 SM ranks before every die-1 SM (a request for <= 4 SMs takes die 0)
    assert max(t["die_packed"][s] for s in range(8) if die[s] == 0) < min(t["die_packed"][s] for s in range(8) if die[s] == 1)
    # die-balanced: any even prefix of ranks holds as many SMs of each die
    inv = sorted(range(8), key=lambda s: t["die_balanced"][s])
    for k in (2, 4, 6, 8):
        assert sum(die[s] for s in inv[:k]) == k // 2
    assert bc._rank_tables(8, None) == {"ascending": list(range(8))}


def _json_lines(stdout):
    out = []
    for line in stdout.splitlines():
        line = line.strip()
        if line.startswith("{"):
            out.append(json.loads(line))
    return out


@pytest.mark.parametrize("n", [1, 2, 4])
def test_bench_launcher_dry_run(n):
    """The real bench.py launcher at N ranks: `--gpus N` re-executes itself under
    torch.distributed.run when no torchrun environment is set, every rank initialises the process
    group (gloo here, no CUDA), partitions the one 512-kernel job queue identically, and rank 0
    alone prints exactly one JSON line with n_gpus = N."""
    env = dict(os.environ)
    for k in ("RANK", "WORLD_SIZE", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT"):
        env.pop(k, None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", str(n), "--dry-run"],
                       capture_output=True, text=True, env=env, timeout=300, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = _json_lines(r.stdout)
    assert len(lines) == 1, r.stdout
    d = lines[0]
    assert d["n_gpus"] == n and d["dry_run"] is True
    assert d["partition_ok"] is True
    assert [x["rank"] for x in d["ranks"]] == list(range(n))
    assert sum(x["kernels"] for x in d["ranks"]) == 512
    assert d["backend"] == (None if n == 1 else "gloo")
    if n > 1:
        busy = [x["predicted_busy_us"] for x in d["ranks"]]
        assert max(busy) / min(busy) < 1.2          # least-backlog assignment balances the GPUs
