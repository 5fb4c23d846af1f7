#!/usr/bin/env python
"""Decompose the runtime-overhead ceiling (SURVEY §8(d) "Runtime-overhead
ceilings"): host spawn rate, GPU-only drain rate (ingest + schedule + dispatch
+ complete, all entries published before launch), overlapped rate, and their
dependence on task size.  Prints one JSON object."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_ppopp_yehsser17_b200 import tasks as T  # noqa: E402
from paper_conf_ppopp_yehsser17_b200.pagoda import NO_START, Pagoda  # noqa: E402


def main():
    out = {}
    N = 60000
    with Pagoda(flags=NO_START, **({"mtbs_per_sm": int(os.environ["MTBS"])} if "MTBS" in os.environ else {})) as p:
        for warps in (1, 4, 8, 16):
            th = 32 * warps
            # pure host spawn into the stopped context
            t0 = time.perf_counter_ns()
            p.spawn_many(N, th, 1, 0, False, T.NOP, None)
            host = (time.perf_counter_ns() - t0) * 1e-9
            # GPU-only: a drain session over the pre-published entries
            t0 = time.perf_counter_ns()
            assert p.start_drain() == 0
            assert p.stop() == 0
            wall = (time.perf_counter_ns() - t0) * 1e-9
            dev = p.session_ms() * 1e-3
            # overlapped: spawn while the session runs
            assert p.start() == 0
            t0 = time.perf_counter_ns()
            p.spawn_many(N, th, 1, 0, False, T.NOP, None)
            assert p.waitAll() == 0
            ov = (time.perf_counter_ns() - t0) * 1e-9
            assert p.stop() == 0
            out[f"nop_w{warps}"] = {"host_spawn_per_s": N / host, "drain_device_per_s": N / dev,
                                    "drain_wall_per_s": N / wall, "overlapped_per_s": N / ov}
    print(json.dumps(out))


if __name__ == "__main__" and len(sys.argv) == 1:
    main()


def ncu_drain(n=60000, threads=128):
    """One self-draining session of n pre-published NOPs (the first launch)."""
    with Pagoda(flags=NO_START) as p:
        p.spawn_many(n, threads, 1, 0, False, T.NOP, None)
        assert p.start_drain() == 0
        assert p.stop() == 0


if __name__ == "__main__" and len(sys.argv) > 1 and sys.argv[1] == "--ncu":
    ncu_drain()
