"""Multi-process host plumbing of the N>1 path on CPU (gloo, world size 2):
the barrier and max/sum-over-ranks reductions bench.py uses around the timed
region, and the reference arm under a 2-rank launch (rank 0 prints one line,
rank 1 exits without work)."""
import json
import os
import time
import socket
import subprocess
import sys

import pytest
import torch.multiprocessing as mp

from conftest import ROOT


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    os.environ.update({"RANK": str(rank), "LOCAL_RANK": str(rank), "WORLD_SIZE": str(world),
                       "MASTER_ADDR": "127.0.0.1", "MASTER_PORT": str(port)})
    sys.path.insert(0, ROOT)
    import bench
    d = bench.Dist()
    d.barrier()
    mx = d.max(float(rank + 1) * 1.5)
    sm = d.sum(float(rank + 1))
    d.barrier()
    q.put((rank, mx, sm))
    import torch.distributed as dist
    dist.destroy_process_group()


def test_gloo_barrier_and_reductions():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    [p.start() for p in procs]
    [p.join(timeout=120) for p in procs]
    assert all(p.exitcode == 0 for p in procs)
    res = sorted(q.get(timeout=5) for _ in range(world))
    assert res == [(0, 3.0, 3.0), (1, 3.0, 3.0)]


@pytest.mark.slow
def test_reference_arm_two_ranks():
    port = _free_port()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.join(ROOT, "bench.py"),
           "--impl", "reference", "--gpus", "2", "--steps", "1", "--warmup", "0", "--workload", "mm"]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["value"] > 0 and d["cpu_baseline"]["kind"] == "oracle"


def _c5_worker(rank, world, port, q):
    """Config 5's strong-scaling shard on each rank (host side: CPU buffers stand in
    for device memory), and the whole-job task count bench.py reports."""
    os.environ.update({"RANK": str(rank), "LOCAL_RANK": str(rank), "WORLD_SIZE": str(world),
                       "MASTER_ADDR": "127.0.0.1", "MASTER_PORT": str(port)})
    sys.path.insert(0, ROOT)
    import bench
    from paper_conf_ppopp_yehsser17_b200 import workloads as W
    d = bench.Dist()
    w = W.c5(10000, device="cpu", pool_size=64, shard=(d.rank, d.world))
    total = d.sum(float(w.n))
    q.put((rank, w.first, w.n, total, int(w.shapes[0, 4])))
    import torch.distributed as dist
    dist.destroy_process_group()


def test_c5_strong_scaling_shards_two_ranks():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_c5_worker, args=(r, world, port, q)) for r in range(world)]
    [p.start() for p in procs]
    [p.join(timeout=300) for p in procs]
    assert all(p.exitcode == 0 for p in procs)
    res = sorted(q.get(timeout=5) for _ in range(world))
    assert [(r[1], r[2]) for r in res] == [(0, 5000), (5000, 5000)]   # disjoint, covering, contiguous
    assert all(r[3] == 10000.0 for r in res)                          # the whole job's tasks on every rank
    from paper_conf_ppopp_yehsser17_b200 import inputs as I
    from paper_conf_ppopp_yehsser17_b200 import workloads as W
    kinds = I.c5_schedule(10000)[0]
    assert res[1][4] == W.KIND_FUNC[I.C5_KINDS[kinds[5000]]]          # rank 1 starts at global task 5000


def _claims_worker(rank, world, port, q):
    """bench.SharedClaims: two ranks claim runs of one step's tasks from the shared counter
    under the least-loaded rule (loads published by each rank); two steps back to back."""
    os.environ.update({"RANK": str(rank), "LOCAL_RANK": str(rank), "WORLD_SIZE": str(world),
                       "MASTER_ADDR": "127.0.0.1", "MASTER_PORT": str(port)})
    sys.path.insert(0, ROOT)
    import bench
    from paper_conf_ppopp_yehsser17_b200 import pagoda as PG
    d = bench.Dist()
    cl = bench.SharedClaims(d, f"test{port}")
    got = []
    n, chunk = 10000, 128
    for step in range(2):
        d.barrier()
        cl.reset(step)
        mine, load = [], 0
        cl.publish(load)
        d.barrier()   # both ranks start claiming together (a late starter would otherwise find nothing left)
        while True:
            cl.publish(load)
            if PG.pool_may_claim(cl.loads(), rank, 4 * chunk) != 1:
                time.sleep(0.002)             # "completions" take time ...
                load = max(0, load - chunk)   # ... and drain this rank's load
                continue
            c = cl.claim(step, chunk, n)
            if c is None:
                break
            mine.append(c)
            load += chunk if rank == 0 else chunk // 2   # rank 1 drains twice as fast: it should claim more
            load = max(0, load - chunk // 2)
        got.append(mine)
    d.barrier()
    cl.close()
    q.put((rank, got))
    import torch.distributed as dist
    dist.destroy_process_group()


def test_shared_claims_two_ranks_cover_each_step_once():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_claims_worker, args=(r, world, port, q)) for r in range(world)]
    [p.start() for p in procs]
    [p.join(timeout=300) for p in procs]
    assert all(p.exitcode == 0 for p in procs)
    res = dict(q.get(timeout=5) for _ in range(world))
    for step in range(2):
        runs = sorted(res[0][step] + res[1][step])
        assert runs == list(range(0, 10000, 128))          # every run of the step claimed exactly once
        assert res[0][step] and res[1][step]               # both ranks took work
