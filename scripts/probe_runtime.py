#!/usr/bin/env python
"""Decompose the runtime-overhead ceiling (SURVEY §8(d) "Runtime-overhead
ceilings"): host spawn rate, GPU-only drain rate (ingest + schedule + dispatch
+ complete, all entries published before launch), overlapped rate, and their
dependence on task size, with the device-side counters of each drain session.
Prints one JSON object.

    python scripts/probe_runtime.py            # the sweep
    python scripts/probe_runtime.py --ncu      # one drain session (for ncu)
    MTBS=1 python scripts/probe_runtime.py     # 1 MTB per SM
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_ppopp_yehsser17_b200 import tasks as T  # noqa: E402
from paper_conf_ppopp_yehsser17_b200.pagoda import NO_START, Pagoda  # noqa: E402


def cfg():
    c = {"flags": NO_START}
    if "MTBS" in os.environ:
        c["mtbs_per_sm"] = int(os.environ["MTBS"])
        if c["mtbs_per_sm"] == 1:
            c["arena_bytes"] = 200 * 1024
    return c


def delta(a, b):
    return {k: b[k] - a[k] for k in b}


def main():
    out = {}
    N = 60000
    with Pagoda(**cfg()) as p:
        for warps in (1, 4, 8, 16):
            th = 32 * warps
            t0 = time.perf_counter_ns()
            p.spawn_many(N, th, 1, 0, False, T.NOP, None)          # pure host spawn, stopped context
            host = (time.perf_counter_ns() - t0) * 1e-9
            c0 = p.counters()
            t0 = time.perf_counter_ns()
            assert p.start_drain() == 0                            # GPU only: everything already published
            assert p.stop() == 0
            wall = (time.perf_counter_ns() - t0) * 1e-9
            dev = p.session_ms() * 1e-3
            cd = delta(c0, p.counters())
            assert p.start() == 0                                  # overlapped: spawn while running
            t0 = time.perf_counter_ns()
            p.spawn_many(N, th, 1, 0, False, T.NOP, None)
            assert p.waitAll() == 0
            ov = (time.perf_counter_ns() - t0) * 1e-9
            assert p.stop() == 0
            out[f"nop_w{warps}"] = {"host_spawn_per_s": N / host, "drain_device_per_s": N / dev,
                                    "drain_wall_per_s": N / wall, "overlapped_per_s": N / ov,
                                    "drain_session_us": dev * 1e6, "drain_counters": cd}
    print(json.dumps(out))


def ncu_drain(n=60000, threads=128):
    """One self-draining session of n pre-published NOPs (the first launch)."""
    with Pagoda(**cfg()) as p:
        p.spawn_many(n, threads, 1, 0, False, T.NOP, None)
        assert p.start_drain() == 0
        assert p.stop() == 0


if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "--ncu":
        ncu_drain()
    else:
        main()
