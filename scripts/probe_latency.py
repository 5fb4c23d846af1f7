"""Spawn-to-done latency (the metric's second half): isolated (one NOP task
in flight, closed loop) and loaded (every task of a 3DES / mix session, per-task
spawn stamp vs a poller's first check()==1), p50/p99 in microseconds.

    python scripts/probe_latency.py > gpurun_out/latency.json
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402

from paper_conf_ppopp_yehsser17_b200 import pagoda as PG  # noqa: E402
from paper_conf_ppopp_yehsser17_b200 import workloads as W  # noqa: E402


def pct(x):
    return {"p50": float(np.percentile(x, 50)), "p99": float(np.percentile(x, 99))}


def main():
    out = {"pingpong_us": pct(PG.pingpong(0, 2000) / 1e3)}
    td = W.tdes(32768, shmem=512)
    mx = W.mix(32768)
    with PG.Pagoda(flags=PG.RESIDENT_TDES | PG.NO_START, arena_bytes=40 * 1024) as p:
        p.tdes_register(td.tdes_tables)
        assert p.start() == 0
        p.latency_loop(200, 128, 1, 0, False, 0)
        out["isolated_nop128_us"] = pct(p.latency_loop(3000, 128, 1, 0, False, 0) / 1e3)
        sp, dn = p.run_timed(td.shapes, td.args)
        out["loaded_tdes_us"] = pct((dn - sp) / 1e3)
        assert p.stop() == 0
    with PG.Pagoda(mtbs_per_sm=1, arena_bytes=200 * 1024) as p:
        sp, dn = p.run_timed(mx.shapes, mx.args)
        out["loaded_mix_us"] = pct((dn - sp) / 1e3)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
