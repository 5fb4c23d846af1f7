#!/usr/bin/env python
"""Does PCIe copy traffic slow the MasterKernel?  3DES session time (config 2)
alone, under a concurrent H2D copy loop, and under a concurrent D2H copy loop.
Prints one JSON object (ms per session)."""
import json
import os
import sys
import threading

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_ppopp_yehsser17_b200 import workloads as W  # noqa: E402
from paper_conf_ppopp_yehsser17_b200.pagoda import NO_START, RESIDENT_TDES, Pagoda  # noqa: E402


def main():
    w = W.tdes(32768)
    nb = 128 << 20
    h = torch.empty(nb, dtype=torch.uint8).pin_memory()
    d = torch.empty(nb, dtype=torch.uint8, device="cuda")
    s = torch.cuda.Stream()
    out = {}
    with Pagoda(flags=NO_START | RESIDENT_TDES, mtbs_per_sm=2, arena_bytes=40 * 1024) as p:
        def step():
            assert p.start() == 0
            p.spawn_shapes(w.shapes, w.args)
            assert p.stop() == 0
            return p.session_ms()
        for mode in ("none", "h2d", "d2h", "none"):
            stop = threading.Event()

            def loop():
                torch.cuda.set_device(0)
                while not stop.is_set():
                    with torch.cuda.stream(s):
                        if mode == "h2d":
                            d.copy_(h, non_blocking=True)
                        else:
                            h.copy_(d, non_blocking=True)
                    s.synchronize()
            th = None
            if mode != "none":
                th = threading.Thread(target=loop, daemon=True)
                th.start()
            for _ in range(2):
                step()
            c0 = p.counters()
            ms = sorted(step() for _ in range(5))
            c1 = p.counters()
            out[mode + "_ctr"] = {k: round((c1[k] - c0[k]) / 5) for k in c1 if c1[k] != c0[k]}
            stop.set()
            if th:
                th.join()
            out[mode] = out.get(mode, []) + [round(ms[2], 3)]
    print(json.dumps(out))


if __name__ == "__main__":
    main()
