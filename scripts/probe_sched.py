#!/usr/bin/env python
"""Where an executor warp's time goes between two tasks, from the trace ledger (PAGODA_TRACE:
allocator events stamped with the low 32 bits of %globaltimer) and the executor intervals.

Per warp and task: body (t_start -> t_end, incl. its fence), then
  end -> folded   the holder folds the warp's free bit (FREE_WARPS event)
  folded -> alloc the warp is given its next task (ALLOC event)
  alloc -> start  wake-up (mbarrier) to the next body start
Reported as medians / means over every warp-gap of one session of the workload at its preset.

    python scripts/probe_sched.py [mm nop tdes]
"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import bench  # noqa: E402
from paper_conf_ppopp_yehsser17_b200 import pagoda as PG  # noqa: E402


def main():
    for name in sys.argv[1:] or ["mm", "nop"]:
        class A:
            workload = name
            no_resident = False
            mtbs = 0
            arena_kb = 0
        cfg = bench.ctx_config(A, PG, name)
        cfg["flags"] |= PG.TRACE
        cfg["trace_events"] = 8192
        w = bench.make_workload(name, bench.use_resident(A, name), bench.Dist())
        n = min(w.n, 65536)
        with PG.Pagoda(**cfg) as p:
            info = p.info()
            if bench.use_resident(A, name) and w.tdes_tables:
                p.tdes_register(w.tdes_tables)
            p.spawn_shapes(w.shapes[:n], w.args[:n])
            assert p.start_drain() == 0
            assert p.stop() == 0
            ms = p.session_ms()
            ev = [p.trace(m) for m in range(info.n_mtb)]
            ex = [[p.exec_trace(m, wp) for wp in range(32)] for m in range(info.n_mtb)]
        gaps = {"end_to_fold": [], "fold_to_alloc": [], "alloc_to_start": [], "body": [], "gap": []}
        for m in range(info.n_mtb):
            e = ev[m]
            if len(e) == 0:
                continue
            t = e["pad2"].astype(np.int64)
            t = np.where(t - t[0] < -(1 << 31), t + (1 << 32), t)   # unwrap the 32-bit stamps
            for wp in range(32):
                x = np.sort(ex[m][wp], order="t_start")
                if len(x) < 2:
                    continue
                bit = 1 << wp
                frees = t[(e["kind"] == 2) & ((e["warp_mask"] & bit) != 0)]
                allocs = t[(e["kind"] == 1) & ((e["warp_mask"] & bit) != 0)]
                ts = (x["t_start"] & 0xFFFFFFFF).astype(np.int64)
                te = (x["t_end"] & 0xFFFFFFFF).astype(np.int64)
                base = t[0]
                ts = np.where(ts - base < -(1 << 31), ts + (1 << 32), ts)
                te = np.where(te - base < -(1 << 31), te + (1 << 32), te)
                for i in range(len(x) - 1):
                    f = frees[(frees >= te[i])]
                    a = allocs[(allocs >= te[i])]
                    if len(f) == 0 or len(a) == 0:
                        continue
                    gaps["end_to_fold"].append(f.min() - te[i])
                    gaps["fold_to_alloc"].append(a.min() - f.min())
                    gaps["alloc_to_start"].append(ts[i + 1] - a.min())
                    gaps["gap"].append(ts[i + 1] - te[i])
                    gaps["body"].append(te[i] - ts[i])
        # concurrency per MTB: time-average number of warps in a body, and the share of the MTB's
        # active span with 0 / 1 / 2 / 3+ tasks in a body (a task is in its body from its first warp's
        # start to its last warp's end)
        warps_busy, occ, span_tot = 0.0, np.zeros(4), 0.0
        for m in range(info.n_mtb):
            recs = [r for wp in range(32) for r in ex[m][wp]]
            if not recs:
                continue
            tid = np.array([r["task_id"] for r in recs], np.int64)
            ts = np.array([int(r["t_start"]) for r in recs], np.int64)
            te = np.array([int(r["t_end"]) for r in recs], np.int64)
            warps_busy += float((te - ts).sum())
            ut = np.unique(tid)
            st = np.array([ts[tid == u].min() for u in ut]); en = np.array([te[tid == u].max() for u in ut])
            t0, t1 = st.min(), en.max()
            span_tot += t1 - t0
            evs = sorted([(x, 1) for x in st] + [(x, -1) for x in en])
            cur, last = 0, t0
            for x, dv in evs:
                occ[min(cur, 3)] += x - last
                cur += dv
                last = x
        out = {"workload": name, "tasks": n, "session_ms": ms, "tasks_per_s": n / ms * 1e3, "mtbs": info.n_mtb,
               "exec_warps_busy_share": warps_busy / (info.n_mtb * info.exec_warps * ms * 1e6),
               "tasks_in_body_share_0_1_2_3plus": [round(float(v / occ.sum()), 3) for v in occ]}
        for k, v in gaps.items():
            v = np.array(v) / 1e3
            out[k] = {"p50_us": float(np.median(v)), "mean_us": float(v.mean()), "n": int(len(v))} if len(v) else None
        print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
