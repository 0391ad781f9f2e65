#!/usr/bin/env python
"""Held-out selector validation shapes (round 2): NEVER fed to
tools/fit_thresholds.py -- they only measure how the fitted table generalises.

  * 5*2^a x 7*2^b and 7*2^a x 5*2^b with a + b = 21 (293 MB) for even a, 22 (587 MB) for odd a,
    a = 1..19: off the power-of-two grid, mostly 16-byte aligned rows;
  * 24 seeded random shapes: R log-uniform in [8, 8M], R*C uniform in [2^26, 2^28] elements
    (256 MiB .. 1 GiB of fp32), so about 3 in 4 have rows off the 16-byte grid.

  python tools/heldout_shapes.py [A|B]      -> "R1xC1,R2xC2,..." for tools/sweep.py --extra
"""
import math
import random


def shapes(which="A"):
    """Set A (round 2, first): 5 / 7 multipliers, seed 20261017 -- after it measured the
    round-1 table (101 / 186 gated shapes passing) it was ADDED to the fit input, so it is no
    longer held out.  Set B: 3 / 13 multipliers, seed 20261018 -- never fitted, but measured in full at
    the end of round 2 and used to FIND the planner rules added then (the rules themselves rest on
    training-set evidence).  Set C: 9 / 11 multipliers, seed 20261021 -- defined after the last
    table and planner change of round 2 and measured once: the clean held-out check."""
    m1, m2, seed = {"A": (5, 7, 20261017), "B": (3, 13, 20261018), "C": (9, 11, 20261021)}[which]
    out = []
    for a in range(1, 20):
        s = 21 if a % 2 == 0 else 22
        out.append((m1 << a, m2 << (s - a)))
        out.append((m2 << a, m1 << (s - a)))
    rng = random.Random(seed)
    for _ in range(24):
        R = int(round(math.exp(rng.uniform(math.log(8), math.log(8 << 20)))))
        E = rng.uniform(1 << 26, 1 << 28)
        C = max(1, int(round(E / R)))
        out.append((R, C))
    return out


def small_shapes(which="Bs"):
    if which == "As":                 # small TRAINING shapes (5 / 7 multipliers, own seed)
        out = []
        for a in range(1, 14):
            s = (14, 15, 17)[a % 3]
            if s - a >= 1:
                out.append((5 << a, 7 << (s - a)))
                out.append((7 << a, 5 << (s - a)))
        rng = random.Random(20261020)
        for _ in range(12):
            R = int(round(math.exp(rng.uniform(math.log(8), math.log(1 << 20)))))
            out.append((R, max(1, int(round(rng.uniform(1 << 20, 1 << 24) / R)))))
        return out
    if which == "Cs":                 # clean small held-out set (round 2, last): 9 / 11 multipliers
        out = []
        for a in range(1, 14):
            s = (14, 15, 17)[a % 3]
            if s - a >= 1:
                out.append((9 << a, 11 << (s - a)))
                out.append((11 << a, 9 << (s - a)))
        rng = random.Random(20261022)
        for _ in range(12):
            R = int(round(math.exp(rng.uniform(math.log(8), math.log(1 << 20)))))
            out.append((R, max(1, int(round(rng.uniform(1 << 20, 1 << 24) / R)))))
        return out
    """Held-out shapes of the paper's small-input regime (4-64 MiB, L2-resident): 3*2^a x
    13*2^b with a + b in {15, 16, 18} (5, 10, 41 MB), and 12 seeded random shapes with R*C
    uniform in [2^20, 2^24] elements.  Never fitted."""
    out = []
    for a in range(1, 15):
        s = (15, 16, 18)[a % 3]
        if s - a >= 1:
            out.append((3 << a, 13 << (s - a)))
            out.append((13 << a, 3 << (s - a)))
    rng = random.Random(20261019)
    for _ in range(12):
        R = int(round(math.exp(rng.uniform(math.log(8), math.log(1 << 20)))))
        E = rng.uniform(1 << 20, 1 << 24)
        out.append((R, max(1, int(round(E / R)))))
    return out


if __name__ == "__main__":
    import sys
    w = sys.argv[1] if len(sys.argv) > 1 else "B"
    print(",".join(f"{R}x{C}" for R, C in (small_shapes(w) if w in ("As", "Bs", "Cs") else shapes(w))))
