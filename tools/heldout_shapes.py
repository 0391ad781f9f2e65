#!/usr/bin/env python
"""Held-out selector validation shapes (round 2): NEVER fed to
tools/fit_thresholds.py -- they only measure how the fitted table generalises.

  * 5*2^a x 7*2^b and 7*2^a x 5*2^b with a + b = 21 (293 MB) for even a, 22 (587 MB) for odd a,
    a = 1..19: off the power-of-two grid, mostly 16-byte aligned rows;
  * 24 seeded random shapes: R log-uniform in [8, 8M], R*C uniform in [2^26, 2^28] elements
    (256 MiB .. 1 GiB of fp32), so about 3 in 4 have rows off the 16-byte grid.

  python tools/heldout_shapes.py            -> "R1xC1,R2xC2,..." for tools/sweep.py --extra
"""
import math
import random


def shapes():
    out = []
    for a in range(1, 20):
        s = 21 if a % 2 == 0 else 22
        out.append((5 << a, 7 << (s - a)))
        out.append((7 << a, 5 << (s - a)))
    rng = random.Random(20261017)
    for _ in range(24):
        R = int(round(math.exp(rng.uniform(math.log(8), math.log(8 << 20)))))
        E = rng.uniform(1 << 26, 1 << 28)
        C = max(1, int(round(E / R)))
        out.append((R, C))
    return out


if __name__ == "__main__":
    print(",".join(f"{R}x{C}" for R, C in shapes()))
