#!/usr/bin/env python
"""A small debug-config run for compute-sanitizer (SURVEY §4 layer 7: racecheck /
synccheck / memcheck "on the debug config (1-2 MTBs, few tasks)").

One MTB with 4 worker warps and an 8-granule arena (the brute-force configuration,
tests/test_gpu_bruteforce.py), plus a 2-SM context (the I/O MTB, its publishers,
forwarders and host poster, and task MTBs): runtime test bodies (MARK, TID, BAR,
SMEM, PAPER) and the paper benchmarks (MB, 3DES, MM, FB, CONV, DCT) are spawned
while stopped, then run by ONE self-draining MasterKernel launch (no host
hand-shake while the sanitizer serialises the kernel).  Exits non-zero if any
task misbehaves.

    compute-sanitizer --tool memcheck  python scripts/sanitize.py
    compute-sanitizer --tool racecheck python scripts/sanitize.py
    compute-sanitizer --tool synccheck python scripts/sanitize.py
"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_ppopp_yehsser17_b200 import tasks as T  # noqa: E402
from paper_conf_ppopp_yehsser17_b200 import workloads as W  # noqa: E402
from paper_conf_ppopp_yehsser17_b200.pagoda import CE_INGEST, NO_START, Pagoda  # noqa: E402


def run(cfg, label, big):
    import torch
    dev = lambda n: torch.zeros(n, dtype=torch.uint8, device="cuda")   # noqa: E731
    err, out, scratch = dev(64), dev(4 * 4096), dev(4 * 4096)
    ws = [W.mandelbrot(2), W.tdes(2, shmem=2560)] + ([W.matmul(2), W.mix(8)] if big else [])
    torch.cuda.synchronize()
    flags = cfg.pop("flags", 0)
    with Pagoda(flags=NO_START | flags, **cfg) as p:
        shapes = [(32, 1, 0, 0, T.NOP, None),
                  (96, 1, 0, 0, T.MARK, np.array([(out.data_ptr(), err.data_ptr() + 32, 0, 7)], T.ARGS[T.MARK])),
                  (64, 2, 0, 0, T.TID, np.array([(out.data_ptr() + 4096, 0, 0)], T.ARGS[T.TID])),
                  (128, 1, 512, 1, T.BAR, np.array([(err.data_ptr(), scratch.data_ptr(), 3, 0)], T.ARGS[T.BAR])),
                  (64, 1, 2048, 1, T.SMEM, np.array([(err.data_ptr() + 4, 2048, 0, 5, 0)], T.ARGS[T.SMEM])),
                  (128, 1, 512, 1, T.PAPER, np.array([(out.data_ptr() + 8192, err.data_ptr() + 8, 0, 0)],
                                                     T.ARGS[T.PAPER]))]
        for th, nb, sh, sy, f, a in shapes:
            assert p.taskSpawn(th, nb, sh, sy, f, a) >= 0
        for w in ws:
            p.spawn_shapes(w.shapes, w.args)
        assert p.start_drain() == 0
        assert p.stop() == 0
        assert p.waitAll() == 0
        info = p.info()
    e = err.cpu().numpy().view(np.uint32)
    assert e[0] == 0 and e[1] == 0 and e[2] == 0 and info.device_error == 0, (label, e[:3], info.device_error)
    print(f"{label}: {info.n_mtb} MTB(s), ok")


def main():
    run({"num_sms": 1, "mtbs_per_sm": 1, "exec_warps": 4, "arena_bytes": 2 * 128 * 64 + 8 * 512}, "debug 1 MTB",
        big=False)
    run({"num_sms": 2, "mtbs_per_sm": 1, "arena_bytes": 200 * 1024}, "2 SMs (I/O MTB + task MTB)", big=True)
    run({"num_sms": 2, "mtbs_per_sm": 1, "arena_bytes": 200 * 1024, "flags": CE_INGEST},
        "2 SMs, copy-engine ingest (scanner warp)", big=True)


if __name__ == "__main__":
    main()
