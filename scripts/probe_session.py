#!/usr/bin/env python
"""Fixed cost vs per-task slope of a self-draining session: session_ms for
N pre-published NOP tasks of w warps, N in {0, 100, 1000, 10000, 60000}.
Prints one JSON object {w: {N: us}}."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_ppopp_yehsser17_b200 import tasks as T  # noqa: E402
from paper_conf_ppopp_yehsser17_b200.pagoda import NO_START, Pagoda  # noqa: E402


def main():
    out = {}
    cfg = {"flags": NO_START}
    if os.environ.get("MTBS") == "1":
        cfg.update(mtbs_per_sm=1, arena_bytes=200 * 1024)
    with Pagoda(**cfg) as p:
        for w in (1, 4, 8):
            row = {}
            for n in (0, 100, 1000, 10000, 60000):
                best = 1e9
                for _ in range(3):
                    if n:
                        p.spawn_many(n, 32 * w, 1, 0, False, T.NOP, None)
                    assert p.start_drain() == 0
                    assert p.stop() == 0
                    best = min(best, p.session_ms() * 1e3)
                row[n] = round(best, 1)
            out[w] = row
    print(json.dumps(out))


if __name__ == "__main__":
    main()
