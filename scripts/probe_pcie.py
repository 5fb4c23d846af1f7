#!/usr/bin/env python
"""PCIe copy bandwidth between pinned host memory and HBM (the e2e floor):
H2D alone, D2H alone, and both at once on two streams.  Prints one JSON line."""
import json

import torch


def main(nbytes=128 << 20, reps=5):
    h_in = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    h_out = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    d_a = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    d_b = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

    def timed(fn):
        best = 1e9
        for _ in range(reps):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            fn()
            torch.cuda.synchronize()
            e1.record()
            torch.cuda.synchronize()
            best = min(best, e0.elapsed_time(e1) * 1e-3)
        return best

    def h2d():
        with torch.cuda.stream(s1):
            d_a.copy_(h_in, non_blocking=True)

    def d2h():
        with torch.cuda.stream(s2):
            h_out.copy_(d_b, non_blocking=True)

    t_h2d = timed(h2d)
    t_d2h = timed(d2h)
    t_both = timed(lambda: (h2d(), d2h()))
    print(json.dumps({"bytes": nbytes, "h2d_gbs": nbytes / t_h2d / 1e9, "d2h_gbs": nbytes / t_d2h / 1e9,
                      "both_ms": t_both * 1e3, "both_gbs_each": nbytes / t_both / 1e9}))


if __name__ == "__main__":
    main()
