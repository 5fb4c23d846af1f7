#!/usr/bin/env python
"""Where a task's time goes between spawn and completion (PAGODA_LIFECYCLE stamps):
for each workload, one warm session then one stamped session of the bench's preset
context; per stage the median / p90 duration (us) and the mean number of tasks in
that stage (Little's law: stage time x throughput).  One JSON line per workload.

    python scripts/probe_life.py [nop mm tdes mix mb]
    PRODUCERS=2 python scripts/probe_life.py mm     # host spawner threads (default: the preset's)
    DRAIN=1 python scripts/probe_life.py mm         # spawn while stopped, then one self-draining session
                                                    # (the device alone: no host spawn in the timed span)
"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import bench  # noqa: E402
from paper_conf_ppopp_yehsser17_b200 import pagoda as PG  # noqa: E402

STAGES = [("ring_wait", 0, 1), ("mtb_queue", 1, 2), ("wake", 2, 3), ("body", 3, 4), ("fence", 4, 5),
          ("post", 5, 6), ("forward", 6, 7), ("pub_to_fwd", 0, 7)]


def main():
    names = sys.argv[1:] or ["nop", "mm", "tdes", "mix", "mb"]
    for name in names:
        class A:
            workload = name
            no_resident = False
            mtbs = 0
            arena_kb = 0
        cfg = bench.ctx_config(A, PG, name)
        cfg["flags"] |= PG.LIFECYCLE
        w = bench.make_workload(name, bench.use_resident(A, name), bench.Dist())
        with PG.Pagoda(**cfg) as p:
            n_mtb = p.info().n_mtb
            if bench.use_resident(A, name) and w.tdes_tables:
                p.tdes_register(w.tdes_tables)
            producers = int(os.environ.get("PRODUCERS", "0")) or bench.PRESETS[name].get("producers", 1)
            drain = os.environ.get("DRAIN") == "1"
            for stamped in (False, True):
                if drain:
                    ids = p.spawn_shapes(w.shapes[:65536], w.args[:65536], ids=True, producers=producers)
                    assert p.start_drain() == 0
                else:
                    assert p.start() == 0
                    ids = p.spawn_shapes(w.shapes, w.args, ids=True, producers=producers)
                assert p.stop() == 0
            ms = p.session_ms()
            L = p.lifecycle(int(ids.min()), len(ids)).astype(np.int64)
        ok = (L > 0).all(axis=1)
        L = L[ok]
        n = len(ids)
        out = {"workload": name, "tasks": n, "stamped": int(ok.sum()), "session_ms": ms,
               "tasks_per_s": n / ms * 1e3, "mtbs": n_mtb, "producers": producers, "drain": drain}
        span = (L[:, 7].max() - L[:, 0].min()) * 1e-9
        rate = len(L) / span
        st = {}
        for nm, a, b in STAGES:
            d = (L[:, b] - L[:, a]) / 1e3
            st[nm] = {"p50_us": float(np.percentile(d, 50)), "p90_us": float(np.percentile(d, 90)),
                      "mean_us": float(d.mean()), "in_stage": float(d.mean() * 1e-6 * rate)}
        out["stages"] = st
        out["span_ms"] = span * 1e3
        print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
