#!/usr/bin/env python
"""Fixed-variant sweep of the five-point stencil on the GPU (second
item): ST_DIRECT and ST_TILE at every super-tile shape TH x TW (and 1/2 CTAs per SM) on
the H x W = 2^k x 2^(e-k) diagonals, one JSON line per run (same format as sweep.py).

The paper picks the super tile by a reuse metric, sum(element accesses) / halo,
constrained by "enough blocks" for small inputs; this sweep measures what the
metric's choice costs against the best tile on B200.

  python tools/sweep_stencil.py --out gpurun_out/sweep_st.jsonl [--elems 22,24,26]
"""
import argparse
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_pldi_samadihmlm12_b200 as adaptic  # noqa: E402
from paper_conf_pldi_samadihmlm12_b200 import _lib as L  # noqa: E402
from tools.sweep import time_plan  # noqa: E402

TH = (4, 8, 16, 32)
TW = (128, 256, 512)


def grid(W):
    out = [("AUTO", None), ("ST_DIRECT", [0, 0, 0, 0, 0, 0, 0, 1]), ("ST_DIRECT", [0, 0, 0, 0, 0, 0, 0, 4])]
    if W >= 4096:
        out.append(("ST_DIRECT", [0, 0, 0, 0, 0, 0, 0, 2]))
    for th in (16, 32, 64, 128):
        out.append(("ST_DIRECT", [0, 0, 0, 0, 0, 0, th, 3]))
    for th in TH:
        for tw in TW:
            if tw > max(128, W):
                continue
            for cps in (0, 1):
                out.append(("ST_TILE", [tw, 0, cps, 0, 0, 0, th]))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", required=True)
    ap.add_argument("--elems", default="22,24,26")
    ap.add_argument("--reps", type=int, default=9)
    ap.add_argument("--kmin", type=int, default=3)
    ap.add_argument("--auto-only", action="store_true")
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    stream = torch.cuda.current_stream().cuda_stream
    shapes = [(1 << k, 1 << (e - k)) for e in (int(v) for v in a.elems.split(","))
              for k in range(a.kmin, e - 6)]
    n = max(H * W for H, W in shapes)
    U = torch.empty(n, device=dev)
    V = torch.empty(n, device=dev)
    coef = torch.tensor([0.6, 0.1], device=dev)
    synth.device_matrix(U, 1, n, "mv", "uniform", 13)
    l2 = torch.cuda.get_device_properties(dev).L2_cache_size
    t0 = time.time()
    with open(a.out, "a") as f:
        for H, W in shapes:
            ptrs = (U.data_ptr(), coef.data_ptr(), V.data_ptr())
            for variant, params in (grid(W) if not a.auto_only else [("AUTO", None)]):
                try:
                    plan = adaptic.get_plan(L.OP_STENCIL5, H, W, L.F32, dev, variant, params, stream)
                except adaptic.AdapticError:
                    continue
                ts = time_plan(plan, ptrs, stream, a.reps)
                med = statistics.median(ts)
                nbytes = 4 * (2 * H * W + 2)
                f.write(json.dumps({"op": "stencil5", "dtype": "f32", "R": H, "C": W, "variant": plan.describe()["variant"],
                                    "req": variant, "params": params, "us": med, "us_min": min(ts),
                                    "GBps": nbytes / med / 1e3, "l2_resident": 8 * H * W < l2,
                                    "plan": plan.describe()}) + "\n")
            adaptic.clear_cache()
            f.flush()
    print(f"stencil sweep done in {time.time() - t0:.1f}s", file=sys.stderr)


if __name__ == "__main__":
    main()
