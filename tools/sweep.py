#!/usr/bin/env python
"""Fixed-variant sweep on the GPU: every variant x parameter grid on every shape.

The paper's compiler estimated break-even points with a performance model
(P:222-232); here they are MEASURED: this tool times each (shape, variant,
params) with CUDA events and writes one JSON line per run; tools/fit_thresholds.py
turns the lines into the selector table (csrc/table_data.inc).

  python tools/sweep.py --out gpurun_out/sweep.jsonl [--elems 26] [--ops mv,tmv] [--dtype f32]
"""
import argparse
import itertools
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

OPC = L.OPS
B1 = ("asum", "nrm2", "iamax", "iamin", "b1all")


CTA_GRID = [(256, rb, u, pp) for rb, u in ((1, 2), (1, 4), (1, 8), (2, 2), (2, 4), (4, 2)) for pp in (1, 2)] + \
           [(1024, 1, 2, 1), (1024, 1, 4, 1), (1024, 2, 2, 1)]


def tile_grid(op, R, C, dtype):
    """The x-tile stream-K kernel (XSMEM 3; fp32 MV on the 128-bit path): chunk widths."""
    if op != "mv" or dtype != "f32" or C % 4 != 0 or C < 512:
        return []
    return [("MV_SPLIT", [cw, 0, 0, 0, 3, 0, 0]) for cw in (0, 8192, 16384) if cw <= C]


def rowtile_grid(op, R, C):
    """Lane groups on TMA-staged row tiles (XSMEM 4; MV/DOT, C <= 32*G): lanes per row G,
    threads per CTA and tile height (rows per ~12 / 24 (auto) / 48 KB of staged data)."""
    if op == "tmv":
        if R > 4096:
            return []
        ok = lambda nt: (R <= nt or (R <= 2 * nt and nt >= 256) or (R <= 4 * nt and nt >= 512)) and \
            (nt != 544 or R <= 1088)  # noqa: E731
        return [("TMV_REGTILE", [0, 0, 0, 0, 4, nt, k]) for nt in (256, 512, 544, 1024) if ok(nt)
                for k in sorted({0, max(4, 12 * 1024 // (4 * R) // 4 * 4), max(4, 48 * 1024 // (4 * R) // 4 * 4)})]
    if op not in ("mv", "dot") or C > 1024:
        return []
    out = []
    opb = 8 if op == "dot" else 4
    for g in (1, 2, 4, 8, 16, 32):
        if C > 32 * g or (g > 1 and C < 2 * g):
            continue
        v = "MV_WPR" if g == 32 else "MV_SUBWARP"
        for nt in (256, 512):
            for kb in (0, 12, 48):
                k = 0 if kb == 0 else max(1, kb * 1024 // (C * opb))
                out.append((v, [g, 0, 0, 0, 4, nt, k]))
    return out


def shift_grid(op, R, C):
    """Misaligned MV rows (C % 4 != 0) with x read from four shifted aligned copies (XSMEM 5)."""
    if op != "mv" or C % 4 == 0 or C < 16:
        return []
    out = []
    nv = C
    if nv <= 256:
        out += [("MV_SUBWARP", [g, 0, 0, u, 5]) for g in (2, 4, 8, 16) for u in (1, 2, 4) if g * u * 4 <= 2 * C]
    if nv <= 16384:
        out += [("MV_WPR", [0, 0, 0, u, 5]) for u in (1, 2, 4, 8) if 32 * u * 4 <= 2 * C]
    if C >= 512:
        out += [("MV_CPR", [nt, 0, 0, u, 5]) for nt, u in ((256, 2), (256, 4), (256, 8), (1024, 2), (1024, 4))]
    if R <= 8192:
        out += [("MV_SPLIT", [nt, 0, 0, u, 5, 0, 0, o]) for nt, u in ((256, 4), (256, 8), (1024, 4)) for o in (1, 2)]
    return out


def misx_grid(op, R, C):
    """Misaligned MV rows, round-2 kernels: x as two aligned loads + a compile-time funnel
    (XSMEM 9) and the shifted-x kernel with RB rows of one residue class (XSMEM 5, ROWS 2/4)."""
    if op != "mv" or C % 4 == 0 or C < 512:
        return []
    out = [("MV_CPR", [256, 0, 0, u, 9]) for u in (2, 4, 8)]
    out += [("MV_CPR", [256, 0, 0, u, 5, 0, rb]) for u in (2, 4) for rb in (2, 4)]
    if R <= 8192:
        out += [("MV_SPLIT", [256, 0, 0, u, 9, 0, 0, o]) for u in (2, 4) for o in (1, 2)]
        out += [("MV_SPLIT", [256, 0, 0, u, 5, 0, rb, o]) for u in (2, 4) for rb in (2, 4) for o in (1, 2)]
    return out


def rtc_grid(op, R, C):
    """Long misaligned MV rows, round 2: k <= 8 whole rows per TMA-staged tile reduced by the
    whole CTA with x in registers (MV_CPR, XSMEM 11); [ctas_per_sm, block, rows (-KB)]."""
    if op != "mv" or C % 4 == 0 or C < 512 or C > 36 * 512:
        return []
    return [("MV_CPR", [0, 0, cps, 0, 11, nt, k]) for nt, k, cps in
            ((256, 0, 0), (256, -48, 0), (512, 0, 0), (512, -48, 0), (512, -48, 2), (256, -48, 2))]


def tshift_grid(op, R, C):
    """TMV rows off the 16-byte grid, round 2: the constant-shift kernel (XSMEM 7; tile width LR,
    c-lanes 256 / LR a multiple of 4, x loads in flight U) and the sliding-window kernel (XSMEM
    10; 4 or 8 rows in flight, splits auto or 1)."""
    if op != "tmv" or R % 4 == 0 or R < 8:
        return []
    return [("TMV_SPLITK", [lr, 0, 0, u, 7]) for lr in (16, 32, 64) for u in (2, 4, 8)] + \
        [("TMV_SPLITK", [0, 0, 0, u, 10]) for u in (4, 8)] + [("TMV_SPLITK", [0, 1, 0, 8, 10])]


def grids(op, R, C, dtype="f32"):
    """(variant, params) candidates; params = [lanes, splits, ctas_per_sm, unroll, xsmem, block, rows], 0 = auto."""
    out = [("AUTO", None)] + tile_grid(op, R, C, dtype) + rowtile_grid(op, R, C) + tshift_grid(op, R, C) + \
        misx_grid(op, R, C) + rtc_grid(op, R, C)
    if op in B1:
        nv = C // 4 if C % 4 == 0 else C
        if nv <= 64:
            for g in (1, 2, 4, 8, 16):
                if g <= max(1, nv):
                    for rb in (1, 4):
                        out.append(("MV_SUBWARP", [g, 0, 0, 0, 0, 0, rb]))
        if nv <= 16384:
            for rb in (1, 4):
                out.append(("MV_WPR", [0, 0, 0, 0, 0, 0, rb]))
        if C >= 256:
            out.append(("MV_CPR", None))
        if R <= 16384:
            for sp in sorted({0} | {max(2, -(-148 * k // R)) for k in (2, 4, 6, 8)}):
                out.append(("MV_SPLIT", [0, sp]))
        return out
    if op in ("mv", "dot"):
        nv = C // 4 if C % 4 == 0 else C
        xms = (1, 2) if op == "mv" and C * 4 <= 200 * 1024 else (0,)
        for xm in xms:
            if nv <= 64:
                for g in (1, 2, 4, 8, 16):
                    if g <= max(1, nv):
                        for u in (1, 2, 4, 8):
                            if g * u <= max(4, 2 * nv):
                                out.append(("MV_SUBWARP", [g, 0, 0, u, xm]))
            if nv <= 8192:
                for u in (1, 2, 4, 8):
                    if 32 * u <= max(32, 2 * nv):
                        out.append(("MV_WPR", [0, 0, 0, u, xm]))
            if C >= 512:
                for nt, rb, u, pp in CTA_GRID:
                    out.append(("MV_CPR", [nt, 0, 0, u, xm, 0, rb, 0, pp]))
        if R <= 8192:
            for nt, rb, u, pp in CTA_GRID:
                for order in (1, 2):
                    out.append(("MV_SPLIT", [nt, 0, 0, u, 0, 0, rb, order, pp]))
        out += shift_grid(op, R, C)
        out += chunk_grid(op, R, C)
        if C <= 256:
            for nt in (128, 256):
                for st in (2, 4, 8):
                    for cps in (0, 1):
                        out.append(("MV_TPR", [nt, 0, cps, st]))
    else:
        rv = R // 4 if R % 4 == 0 else R
        for u in (2, 4, 8):
            out.append(("TMV_COL", [0, 0, 0, u]))
        for nt in (256, 1024):
            for lr in (1, 2, 4, 8, 16, 32, 64, 128, 256):
                if lr > max(1, 2 * rv) or (rv >= 4096 and lr < 8):
                    continue
                tiles = -(-rv // lr)
                splits = sorted({0} | {max(1, -(-148 * k // tiles)) for k in (1, 2, 4, 8)})
                for u in ((2, 4, 8) if nt == 256 else (2, 4)):
                    for sp in splits:
                        if sp > C:
                            continue
                        out.append(("TMV_SPLITK", [lr, sp, 0, u, 0, nt]))
        for u in (2, 4, 8):
            out.append(("TMV_REGTILE", [0, 0, 0, u]))
    return out


def chunk_grid(op, R, C):
    """MV rows on staged column chunks (XSMEM 13, round 2; any C, any alignment): x values per
    thread MX and threads NT (chunk width <= NT MX), row segments per tile (0: ~64 KB)."""
    if op != "mv" or C < 8192:
        return []
    return [("MV_SPLIT", [mx, 0, 0, 0, 13, nt, k]) for mx, nt in ((16, 512), (36, 512), (36, 256))
            for k in (0, 1, 2, 4)]


def time_plan(plan, ptrs, stream, reps, batch=5, graph=False):
    """Per-launch time of back-to-back launches (the way bench.py and a stream of
    calls see it): `reps` samples, each = CUDA-event time of `batch` launches / batch.
    graph=True (small, L2-resident problems, round 2): the launches are replayed from a CUDA
    graph of 20, so the sample is device time, not the host's launch rate (~5 us per
    ctypes launch, which had made every candidate of a <= 64 MiB shape look alike)."""
    for _ in range(2):
        plan.run(*ptrs, stream)
    torch.cuda.synchronize()
    if graph:
        n = 20
        s = torch.cuda.Stream()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.stream(s):
            plan.run(*ptrs, s.cuda_stream)
            torch.cuda.synchronize()
            with torch.cuda.graph(g, stream=s):
                for _ in range(n):
                    plan.run(*ptrs, torch.cuda.current_stream().cuda_stream)
            g.replay()
            torch.cuda.synchronize()
            out = []
            for _ in range(reps):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(s)
                g.replay()
                b.record(s)
                b.synchronize()
                out.append(a.elapsed_time(b) * 1e3 / n)
        return out
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for a, b in evs:
        a.record()
        for _ in range(batch):
            plan.run(*ptrs, stream)
        b.record()
    torch.cuda.synchronize()
    return [a.elapsed_time(b) * 1e3 / batch for a, b in evs]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", required=True)
    ap.add_argument("--elems", default="26", help="comma list of log2(R*C) diagonals")
    ap.add_argument("--ops", default="mv,tmv")
    ap.add_argument("--dtype", default="f32")
    ap.add_argument("--reps", type=int, default=9)
    ap.add_argument("--kmin", type=int, default=3)
    ap.add_argument("--kmax", type=int, default=23)
    ap.add_argument("--extra", default="", help="extra shapes R1xC1,R2xC2")
    ap.add_argument("--perturb", action="store_true",
                    help="also time each diagonal shape with the reduction length (MV/DOT: C+1) or the "
                         "output count (TMV: R+1) off the 128-bit path, for the scalar-shape table cells")
    ap.add_argument("--perturb-only", action="store_true", help="only the perturbed (off-128-bit-path) shapes")
    ap.add_argument("--auto-only", action="store_true", help="time only the selector's pick (validation runs)")
    ap.add_argument("--tile-only", action="store_true", help="time only the x-tile stream-K candidates (+ AUTO)")
    ap.add_argument("--rowtile-only", action="store_true", help="time only the staged row-tile candidates (+ AUTO)")
    ap.add_argument("--flat-only", action="store_true", help="time only the flat-stream TMV candidates (+ AUTO)")
    ap.add_argument("--shift-only", action="store_true", help="time only the shifted-x MV candidates (+ AUTO)")
    ap.add_argument("--staged-only", action="store_true", help="time only the TMA-staged candidates (+ AUTO)")
    ap.add_argument("--tshift-only", action="store_true", help="time only the constant-shift TMV candidates (+ AUTO)")
    ap.add_argument("--misx-only", action="store_true", help="time only the round-2 misaligned-MV candidates (+ AUTO)")
    ap.add_argument("--rtc-only", action="store_true", help="time only the long-row staged MV candidates (+ AUTO)")
    ap.add_argument("--chunk-only", action="store_true", help="time only the column-chunk staged MV candidates (+ AUTO)")
    ap.add_argument("--graph-below", type=float, default=0,
                    help="time problems smaller than this many bytes from CUDA graphs (device time)")
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    tdt = torch.float32 if a.dtype == "f32" else torch.int32
    dtc = L.F32 if a.dtype == "f32" else L.I32
    stream = torch.cuda.current_stream().cuda_stream
    shapes = []
    for e in (int(v) for v in a.elems.split(",")):
        for k in range(a.kmin, min(a.kmax, e - 3) + 1):
            shapes.append((1 << k, 1 << (e - k)))
    for s in filter(None, a.extra.split(",")):
        r, c = s.lower().split("x")
        shapes.append((int(r), int(c)))
    if a.perturb_only:
        shapes = [(R, C, 1) for R, C in shapes]
    elif a.perturb:
        shapes = [(R, C, p) for R, C in shapes for p in (0, 1)]
    else:
        shapes = [(R, C, 0) for R, C in shapes]
    maxel = max(R * C for R, C, _ in shapes) + max(R + C for R, C, _ in shapes)
    M = torch.empty(maxel * (2 if "dot" in a.ops else 1) + 64, dtype=tdt, device=dev)
    X = torch.empty(max(C for _, C, _ in shapes) + 1, dtype=tdt, device=dev)
    Y = torch.empty(4 * (max(R for R, _, _ in shapes) + 1), dtype=tdt, device=dev)   # 4-byte y; B1ALL: 4 per row
    synth.device_matrix(M, 1, M.numel(), "mv", "uniform", 11)
    synth.device_vector(X, "uniform", 12)
    t0 = time.time()
    with open(a.out, "a") as f:
        for op in a.ops.split(","):
            for R0, C0, pert in shapes:
                R, C = (R0 + pert, C0) if op == "tmv" else (R0, C0 + pert)
                # DOT's b: 256-byte aligned like a separate allocation (round 1 placed it right
                # after a, so a and b differed in address mod 16 whenever R*C % 4 != 0 and the
                # misaligned-row DOT kernels -- which need equal alignment -- fell back to scalar)
                Xp = M.data_ptr() + (R * C * 4 + 255) // 256 * 256 if op == "dot" else X.data_ptr()
                ptrs = (M.data_ptr(), Xp, Y.data_ptr())
                if a.auto_only:
                    cands = [("AUTO", None)]
                elif a.tile_only:
                    cands = [("AUTO", None)] + tile_grid(op, R, C, a.dtype)
                elif a.rowtile_only:
                    cands = [("AUTO", None)] + rowtile_grid(op, R, C)
                elif a.shift_only:
                    cands = [("AUTO", None)] + shift_grid(op, R, C)
                elif a.staged_only:           # every TMA-staged plan: row tiles, TMV tiles, MV_TPR
                    cands = [("AUTO", None)] + rowtile_grid(op, R, C) + \
                        [c for c in grids(op, R, C, a.dtype) if c[0] == "MV_TPR"]
                elif a.misx_only:
                    cands = [("AUTO", None)] + misx_grid(op, R, C)
                elif a.rtc_only:
                    cands = [("AUTO", None)] + rtc_grid(op, R, C)
                elif a.chunk_only:
                    cands = [("AUTO", None)] + chunk_grid(op, R, C)
                elif a.tshift_only:
                    cands = [("AUTO", None)] + tshift_grid(op, R, C)
                elif a.flat_only:
                    cands = [("AUTO", None)] + [("TMV_REGTILE", [0, 0, 0, u]) for u in (2, 4, 8)] + \
                        rowtile_grid(op, R, C)
                else:
                    cands = grids(op, R, C, a.dtype)
                for variant, params in cands:
                    try:
                        plan = adaptic.get_plan(OPC[op], R, C, dtc, dev, variant, params, stream)
                    except adaptic.AdapticError:
                        continue
                    nbytes = 4 * (R * C * (2 if op == "dot" else 1) + (4 if op == "b1all" else 1) * R
                                  + (0 if op in ("dot",) + B1 else C))
                    ts = time_plan(plan, ptrs, stream, a.reps, graph=nbytes < a.graph_below)
                    med = statistics.median(ts)
                    d = plan.describe()
                    f.write(json.dumps({"op": op, "dtype": a.dtype, "R": R, "C": C, "variant": d["variant"],
                                        "req": variant, "params": params, "us": med, "us_min": min(ts),
                                        "timing": "graph" if nbytes < a.graph_below else "stream",
                                        "GBps": nbytes / med / 1e3, "plan": d}) + "\n")
                adaptic.clear_cache()
                f.flush()
    print(f"sweep done in {time.time() - t0:.1f}s", file=sys.stderr)


if __name__ == "__main__":
    main()
