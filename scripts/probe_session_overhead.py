"""Fixed cost of one MasterKernel session (launch -> exit, CUDA events on its
stream) with 0 and 1 tasks, per context configuration.

    python scripts/probe_session_overhead.py
"""
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_ppopp_yehsser17_b200 import pagoda as PG  # noqa: E402


def main():
    out = {}
    for name, cfg in {"2mtb_96k": {}, "2mtb_res40k": {"flags": PG.RESIDENT_TDES, "arena_bytes": 40 * 1024},
                      "1mtb_200k": {"mtbs_per_sm": 1, "arena_bytes": 200 * 1024}}.items():
        flags = PG.NO_START | cfg.pop("flags", 0)
        p = PG.Pagoda(flags=flags, **cfg)
        for n in (0, 1):
            dev, host = [], []
            for i in range(12):
                t0 = time.perf_counter_ns()
                assert p.start() == 0
                if n:
                    p.taskSpawn(128, 1, 0, False, 0)
                assert p.stop() == 0
                host.append((time.perf_counter_ns() - t0) / 1e3)
                dev.append(p.session_ms() * 1e3)
            out[f"{name}_tasks{n}"] = {"device_us_p50": statistics.median(dev[2:]),
                                       "host_us_p50": statistics.median(host[2:])}
        p.shutdown()
    print(json.dumps(out))


if __name__ == "__main__":
    main()
