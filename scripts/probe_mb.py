#!/usr/bin/env python
"""Where does config 1 (Mandelbrot, 1024 tiles) spend its session?  Runs one
traced drain session and reports per-task durations, the SM each task ran on,
saturated tiles per SM, and the session's critical path.  One JSON line."""
import json
import os
import sys
from collections import Counter, defaultdict

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_ppopp_yehsser17_b200 import workloads as W  # noqa: E402
from paper_conf_ppopp_yehsser17_b200.pagoda import NO_START, TRACE, Pagoda  # noqa: E402


def main():
    mtbs = int(os.environ.get("MTBS", "2"))
    w = W.mandelbrot(1024)
    cfg = dict(flags=NO_START | TRACE, trace_events=4096, mtbs_per_sm=mtbs)
    if mtbs == 1:
        cfg["arena_bytes"] = 200 * 1024
    with Pagoda(**cfg) as p:
        p.spawn_shapes(w.shapes, w.args)
        assert p.start_drain() == 0
        assert p.stop() == 0
        sess_us = p.session_ms() * 1e3
        info = p.info()
        recs = np.concatenate([p.exec_trace(m, k) for m in range(info.n_mtb) for k in range(32)])
    out = w.outputs()["out"].reshape(1024, -1).astype(np.int64)
    cost = out.sum(1)                          # iterations per tile
    sat = set(np.nonzero((out == 256).all(1))[0].tolist())
    t0 = recs["t_start"].min()
    task = defaultdict(lambda: [1 << 62, 0, -1])
    for r in recs:
        t = task[int(r["task_id"])]
        t[0] = min(t[0], int(r["t_start"]))
        t[1] = max(t[1], int(r["t_end"]))
        t[2] = int(r["smid"])
    dur = {k: (v[1] - v[0]) / 1e3 for k, v in task.items()}
    sm_sat = Counter(v[2] for k, v in task.items() if k in sat)
    sm_tasks = Counter(v[2] for v in task.values())
    last = max(v[1] for v in task.values())
    res = {"session_us": sess_us, "first_start_to_last_end_us": (last - t0) / 1e3,
           "tasks": len(task), "sms_used": len(sm_tasks),
           "sat_task_us_p50": float(np.median([dur[k] for k in sat if k in dur])),
           "sat_task_us_max": float(max(dur[k] for k in sat if k in dur)),
           "cheap_task_us_p50": float(np.median([d for k, d in dur.items() if k not in sat])),
           "max_sat_per_sm": max(sm_sat.values()), "sms_with_ge2_sat": sum(1 for v in sm_sat.values() if v >= 2),
           "max_tasks_per_sm": max(sm_tasks.values()),
           "last_task_start_us": (max(v[0] for v in task.values()) - t0) / 1e3,
           "total_iterations": int(cost.sum())}
    print(json.dumps(res))


if __name__ == "__main__":
    main()
