"""NEXT-3 sweeps on one GPU, one JSON object per point:

  tasks   : #tasks in {32 .. 32768} of 3DES (4 KiB, 128 threads)   (Fig. 6)
  threads : threads per task in {32 .. 1024}, 32768 3DES tasks      (Fig. 7)
            and 8192 MB tiles (MB repeats config 1's 1024 tiles)
  large   : 4096 CONV tasks (128x128) of 128 .. 16384 threads; above 1024 the task is
            several 1024-thread TBs spread over MTBs (Fig. 8's large tasks)
  size    : input size x threads (Fig. 8): 3DES packets of 1 .. 64 KiB with
            64 .. 512 threads per task, 64 MiB of packets per point (65536 .. 1024 tasks)

    python scripts/sweeps.py [tasks threads large size]   # default: all

Each point: Pagoda (one session: start -> spawn all -> stop; CUDA-event
device time and host time), the naive one-launch-per-task baseline and the
static-fusion kernel (256 threads per task).  Parity of every body is the
job of tests/; this script only times.

    python scripts/sweeps.py > gpurun_out/sweeps.jsonl
"""
import json
import os
import statistics
import sys
import time

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_ppopp_yehsser17_b200 import pagoda as PG  # noqa: E402
from paper_conf_ppopp_yehsser17_b200 import workloads as W  # noqa: E402


def time_pagoda(w, reps=5, **cfg):
    p = PG.Pagoda(flags=PG.NO_START | cfg.pop("flags", 0), **cfg)
    dev, host = [], []
    for i in range(reps + 2):
        t0 = time.perf_counter_ns()
        assert p.start() == 0
        p.spawn_shapes(w.shapes, w.args)
        assert p.stop() == 0
        if i >= 2:
            host.append((time.perf_counter_ns() - t0) * 1e-9)
            dev.append(p.session_ms() * 1e-3)
    assert p.shutdown() == 0
    return w.n / statistics.median(dev), w.n / statistics.median(host)


def time_naive(w):
    PG.naive_run(0, w.shapes[:256], w.args[:256], 32)
    return w.n / (statistics.median(PG.naive_run(0, w.shapes, w.args, 32) for _ in range(2)) * 1e-9)


def time_fused(w):
    if (w.shapes[:, 1] != 1).any():
        return None   # static fusion runs one thread block per task
    PG.fused_run(0, w.shapes[:256], w.args[:256], 256)
    r = [PG.fused_run(0, w.shapes, w.args, 256) for _ in range(3)]
    return w.n / (statistics.median(x[0] for x in r) * 1e-9)


def point(sweep, label, w, **cfg):
    dev, host = time_pagoda(w, **cfg)
    out = {"sweep": sweep, **label, "n_tasks": w.n, "pagoda_tasks_per_s": dev, "pagoda_host_tasks_per_s": host,
           "naive_tasks_per_s": time_naive(w), "fused_tasks_per_s": time_fused(w)}
    out["speedup_vs_naive"] = dev / out["naive_tasks_per_s"]
    out["speedup_vs_fused"] = dev / out["fused_tasks_per_s"] if out["fused_tasks_per_s"] else None
    print(json.dumps(out), flush=True)


def main():
    torch.cuda.set_device(0)
    which = set(sys.argv[1:]) or {"tasks", "threads", "large", "size"}
    res = {"flags": PG.RESIDENT_TDES, "arena_bytes": 40 * 1024}
    if "tasks" in which:
        for n in (32, 128, 512, 2048, 8192, 32768):   # Fig. 6: the number of tasks
            w = W.tdes(n, shmem=512)
            point("tasks", {"body": "tdes", "threads": 128}, w, **res)
    if "threads" in which:
        for th in (32, 64, 128, 256, 512, 1024):       # Fig. 7: threads per task
            w = W.tdes(32768, shmem=512, threads=th)
            point("threads", {"body": "tdes", "threads": th}, w, **res)
            w = W.mandelbrot(8192, threads=th)
            point("threads", {"body": "mb", "threads": th}, w)
    if "large" in which:
        for th in (128, 512, 1024, 4096, 16384):       # Fig. 8: large tasks, spread over MTBs above 1024
            w = W.conv_only(4096, threads=min(th, 1024), n_tb=max(1, th // 1024))
            point("large", {"body": "conv", "threads": th, "tbs": max(1, th // 1024)}, w)
    if "size" in which:
        for kib in (1, 4, 16, 64):                     # Fig. 8: input size x threads, 64 MiB per point
            for th in (64, 128, 256, 512):
                w = W.tdes((64 << 20) // (kib << 10), nbytes=kib << 10, threads=th, shmem=512)
                point("size", {"body": "tdes", "packet_kib": kib, "threads": th}, w, **res)
                del w
                torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
