"""Executor busy fraction from the trace (SURVEY §8(d) ncu evidence: "executor
busy fraction = sum of body warp-time / (executor warps x elapsed)"), plus the
median body duration and the median idle gap between two tasks on a warp.
PAGODA_TRACE slows scheduling a little; the fractions are what matter.

    python scripts/probe_busy.py [mm tdes mb ...] > gpurun_out/busy.json
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402

from paper_conf_ppopp_yehsser17_b200 import pagoda as PG  # noqa: E402
from paper_conf_ppopp_yehsser17_b200 import workloads as W  # noqa: E402


def probe(name):
    if name == "tdes":
        w, cfg = W.tdes(32768, shmem=512), {"flags": PG.RESIDENT_TDES, "arena_bytes": 40 * 1024}
    elif name == "mm":
        w, cfg = W.matmul(65536), {}
    elif name == "mb":
        w, cfg = W.mandelbrot(1024), {}
    else:
        w, cfg = W.nop(65536, threads=256), {}
    cfg["flags"] = cfg.get("flags", 0) | PG.TRACE
    with PG.Pagoda(trace_events=4096, **cfg) as p:
        p.spawn_shapes(w.shapes, w.args)
        assert p.waitAll() == 0
        info = p.info()
        recs = []
        for m in range(info.n_mtb):
            for wp in range(32):
                r = p.exec_trace(m, wp)
                if len(r):
                    recs.append(r)
    allr = np.concatenate(recs)
    t0, t1 = int(allr["t_start"].min()), int(allr["t_end"].max())
    busy = float((allr["t_end"] - allr["t_start"]).sum())
    n_warps = sum(1 for _ in recs)
    gaps = np.concatenate([np.diff(np.sort(r["t_start"]))[:] - (r["t_end"] - r["t_start"])[np.argsort(r["t_start"])][:-1]
                           for r in recs if len(r) > 1])
    per_mtb = {}
    for r in recs:
        per_mtb[int(r["mtb"][0])] = per_mtb.get(int(r["mtb"][0]), 0) + len(r)
    return {"workload": name, "tasks": w.n, "span_us": (t1 - t0) / 1e3, "warps_used": n_warps,
            "busy_frac": busy / (n_warps * (t1 - t0)),
            "body_us_p50": float(np.median(allr["t_end"] - allr["t_start"])) / 1e3,
            "gap_us_p50": float(np.median(gaps)) / 1e3, "gap_us_p90": float(np.percentile(gaps, 90)) / 1e3,
            "warp_tasks_per_mtb_min_max": [min(per_mtb.values()), max(per_mtb.values())]}


if __name__ == "__main__":
    for name in sys.argv[1:] or ["mm", "tdes", "nop"]:
        print(json.dumps(probe(name)), flush=True)
