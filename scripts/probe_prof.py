"""Where the MasterKernel's time goes (profiling build: PAGODA_LIB=build/variants/libpagoda_vprof.so):
scheduler-holder phases and executor steps, in ns per task and as a share of the MTBs' time.

    PAGODA_LIB=... python scripts/probe_prof.py > gpurun_out/prof.json
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_ppopp_yehsser17_b200 import pagoda as PG  # noqa: E402
from paper_conf_ppopp_yehsser17_b200 import workloads as W  # noqa: E402


def run(name, w, **cfg):
    p = PG.Pagoda(flags=PG.NO_START | cfg.pop("flags", 0), **cfg)
    for _ in range(2):
        assert p.start() == 0
        p.spawn_shapes(w.shapes, w.args)
        assert p.stop() == 0
    c0 = p.counters()
    assert p.start() == 0
    p.spawn_shapes(w.shapes, w.args)
    assert p.stop() == 0
    ms = p.session_ms()
    c = {k: v - c0[k] for k, v in p.counters().items()}
    n_mtb = p.info().n_mtb
    p.shutdown()
    out = {"workload": name, "tasks": w.n, "session_ms": ms, "tasks_per_s": w.n / ms * 1e3,
           "ns_per_task": {k: c[k] / w.n for k in c if "_ns_" in k},
           "mtb_time_share": {k: c[k] / (n_mtb * ms * 1e6) for k in c if k.startswith("sched_ns")},
           "counts_per_task": {k: c[k] / w.n for k in ("sched_rounds", "tickets", "claim_empty", "load_not_ready",
                                                       "place_nofit", "handoffs")}}
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    run("nop4", W.nop(65536, threads=128))
    run("nop8", W.nop(65536, threads=256))
    run("mm", W.matmul(65536))
    run("mm_4mtb", W.matmul(65536), mtbs_per_sm=4, arena_bytes=48 * 1024)
    run("tdes", W.tdes(32768, shmem=512), flags=PG.RESIDENT_TDES, arena_bytes=40 * 1024)
