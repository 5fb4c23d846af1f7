"""Generate tests/golden/mandelbrot_pins.txt — the Mandelbrot (config 1) pins.

An INDEPENDENT float32 emulation of the MB definition (SURVEY §8(c) "MB",
DESIGN.md "Task bodies"; P:1031-1032 names the benchmark, BASELINE.json
configs[0] fixes 1024 tiles of 64x64 and 256 iterations).  It uses numpy only:
no code from oracle/ or from the CUDA product.  numpy rounds every float32
operation separately (it never contracts a*b+c into an fma), which is exactly
the definition's "mul then add, not fused":

    cr = -2 + gx * (3/2048),  ci = -1.5 + gy * (3/2048)    (exact in fp32)
    zr = zi = 0, n = 0
    while n < 256:
        zr2 = zr*zr; zi2 = zi*zi
        if zr2 + zi2 > 4: break         (strict '>')
        t = zr + zr; zi = t*zi + ci; zr = (zr2 - zi2) + cr; n += 1

    python scripts/gen_mandelbrot_pins.py            # rewrite the golden file
    python scripts/gen_mandelbrot_pins.py --check    # compare with it (exit 1 on a difference)

tests/test_oracle_bodies.py::test_mb_golden_file_regenerates runs --check's logic.
"""
from __future__ import annotations

import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = os.path.join(ROOT, "tests", "golden", "mandelbrot_pins.txt")
N, TILE, MAXIT = 2048, 64, 256
PIXELS = [(0, 1024), (1024, 1024), (1536, 1024), (1536, 1536)]   # (gx, gy)

HEADER = """\
# Mandelbrot pins for config 1 (SURVEY §8(c) MB; BASELINE.json configs[0]).
# Grid: cr = -2 + gx*3/2048, ci = -1.5 + gy*3/2048, 2048x2048 pixels = 32x32 tiles of 64x64, maxit 256.
# Written by scripts/gen_mandelbrot_pins.py: an independent numpy float32 emulation (per-op rounding,
# no fma), sharing no code with oracle/ or the CUDA product.  SURVEY.md §8(c) "Pins" quotes the same values.
# (0,1024) is c = -2: the orbit -2 -> 2 -> 2 ... has |z|^2 = 4 exactly, so '>=' would give 1 (tie-break pin).
# c = 0.25+0.75i -> 5 is also derivable by hand: z1=.25+.75i, z2=-.25+1.125i, z3=-.953125+.1875i,
# z4=1.123291015625+.392578125i, |z5|^2 ~ 4.51 > 4.
# format: gx gy count
"""


def iteration_counts(fused: bool = False) -> np.ndarray:
    """counts[gy, gx] for the whole 2048x2048 grid.  fused=True contracts the two
    multiply-adds instead (fp64 evaluation, one rounding to fp32): the variant the
    definition forbids, used only to show that the pins detect it."""
    f = np.float32
    g = np.arange(N, dtype=np.float32)
    cr_row = (f(-2.0) + g * f(3.0 / 2048)).astype(np.float32)
    ci_col = (f(-1.5) + g * f(3.0 / 2048)).astype(np.float32)
    cr = np.broadcast_to(cr_row[None, :], (N, N)).reshape(-1).copy()
    ci = np.broadcast_to(ci_col[:, None], (N, N)).reshape(-1).copy()
    idx = np.arange(N * N)
    counts = np.full(N * N, MAXIT, np.int32)   # pixels never escaping keep 256
    zr = np.zeros(N * N, np.float32)
    zi = np.zeros(N * N, np.float32)
    four = f(4.0)
    for n in range(MAXIT):
        zr2 = zr * zr
        zi2 = zi * zi
        esc = (zr2 + zi2) > four
        if esc.any():
            counts[idx[esc]] = n
            keep = ~esc
            idx, zr, zi, zr2, zi2, cr, ci = (a[keep] for a in (idx, zr, zi, zr2, zi2, cr, ci))
        t = zr + zr
        if fused:
            zi = (t.astype(np.float64) * zi + ci).astype(np.float32)
        else:
            zi = t * zi + ci
        zr = (zr2 - zi2) + cr
    return counts.reshape(N, N)


def render(counts: np.ndarray) -> str:
    tiles = counts.reshape(N // TILE, TILE, N // TILE, TILE).sum(axis=(1, 3), dtype=np.int64).reshape(-1)
    lines = [HEADER]
    for gx, gy in PIXELS:
        lines.append(f"{gx} {gy} {int(counts[gy, gx])}\n")
    lines.append("# whole-config facts\n")
    lines.append(f"# sum {int(counts.sum(dtype=np.int64))}\n")
    lines.append(f"# saturated_tiles {int((tiles == TILE * TILE * MAXIT).sum())}\n")
    lines.append(f"# tile_sum_min {int(tiles.min())}\n")
    med = float(np.median(tiles))
    lines.append(f"# tile_sum_median {med:g}\n" if med != int(med) else f"# tile_sum_median {int(med)}\n")
    lines.append(f"# tile_sum_max {int(tiles.max())}\n")
    return "".join(lines)


def main(argv) -> int:
    text = render(iteration_counts())
    if "--check" in argv:
        with open(GOLDEN) as f:
            ok = f.read() == text
        print("golden file matches" if ok else "golden file DIFFERS")
        return 0 if ok else 1
    with open(GOLDEN, "w") as f:
        f.write(text)
    print("wrote", GOLDEN)
    return 0


if __name__ == "__main__":
    sys.exit(main(sys.argv[1:]))
