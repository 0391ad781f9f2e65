#!/usr/bin/env python
"""Fit the selector table from measured sweeps (tools/sweep.py JSONL).

The paper splits the input range into subranges at the performance model's
break-even points and generates one kernel per subrange (Fig. 2).
Here the "model" is the measurement itself: for every measured cell
(op, dtype, floor(log2 R), floor(log2 C)) the fastest (variant, params) becomes
that cell's entry; the planner (csrc/adaptic.cu) uses the nearest cell for
unmeasured shapes.  Tie-break (deterministic): runs within 1 % of the
fastest are equivalent; among them prefer the one with fewer CTAs.

  python tools/fit_thresholds.py gpurun_out/sweep*.jsonl --ops mv,tmv,dot \
      --out paper_conf_pldi_samadihmlm12_b200/csrc/table_data.inc --json profiles/selector_table.json
  python tools/fit_thresholds.py gpurun_out/sweep_blas1*.jsonl --ops asum,nrm2,iamax,iamin \
      --out paper_conf_pldi_samadihmlm12_b200/csrc/table_b1.inc --json profiles/selector_table_b1.json
"""
import argparse
import collections
import json
import math

VARIANT_ID = {"MV_TPR": 1, "MV_SUBWARP": 2, "MV_WPR": 3, "MV_CPR": 4, "MV_SPLIT": 5,
              "TMV_COL": 6, "TMV_SPLITK": 7, "TMV_REGTILE": 8}
OP_ID = {"mv": 0, "tmv": 1, "dot": 2, "asum": 3, "nrm2": 4, "iamax": 5, "iamin": 6, "b1all": 7}
DT_ID = {"f32": 0, "i32": 1}


def norm_params(r):
    """Cell-portable parameters: a staged-tile plan's explicit tile height (rows of the
    measured shape) becomes a tile SIZE, -KB (derive() reads ROWS < 0 as kilobytes), so the
    entry means the same thing for every shape of its cell."""
    p = list(r["params"] or []) + [0] * 9
    if p[4] in (4, 11) and p[6] > 0:
        if r["op"] == "tmv":
            row_bytes = 4 * (r["R"] + 1)
        else:
            row_bytes = 4 * r["C"] * (2 if r["op"] == "dot" else 1)
        p[6] = -max(1, math.ceil(p[6] * row_bytes / 1024))     # whole KB, rounded up: derive() floors back to the rows
    return p[:9]


def fit(rows, tie=0.01, protect=None, protect_tol=0.01, neighbor_weight=0.0, portable_tie=0.0, prefer_staged_dot=0.0):
    """Per cell (op, dtype, load-path class, floor(log2 R), floor(log2 C)): the candidate
    (variant, portable params) with the best mean fraction of each shape's best GB/s over
    the cell's measured shapes (a cell may hold a diagonal shape and held-out ones of other
    sizes, so raw times are not comparable; a shape a candidate was not run on counts at
    the candidate's own mean less 3 %).  Ties within 1 %: fewer CTAs.

    protect: (op, R, C) shapes whose cell pick must stay within protect_tol of the best
    measured run ON THAT SHAPE (the benchmark's own shapes): in a cell holding one, only
    such candidates compete, and the cell's other shapes decide among them.

    neighbor_weight: the shapes of the adjacent cells (Manhattan distance 1, same op, dtype
    and load class) also score a candidate, with this weight -- a pick is used for unmeasured
    shapes around its cell too, so one that only fits its own shapes generalises badly.
    portable_tie: among candidates within this fraction of the top score, prefer the one
    with the most planner-derived (0) parameters (they adapt to the actual shape)."""
    cells = collections.defaultdict(list)
    for r in rows:
        if r["req"] == "AUTO":
            continue
        vec = 1 if r["plan"]["vec_shape"] else 0      # 128-bit path shape (C % 4 == 0; TMV: R % 4 == 0)
        cells[(r["op"], r["dtype"], vec, int(math.log2(r["R"])), int(math.log2(r["C"])))].append(r)
    def cell_cands(rs):
        best = {}
        cand = collections.defaultdict(dict)          # (variant, params) -> shape -> best run
        for r in rs:
            sh = (r["R"], r["C"])
            best[sh] = max(best.get(sh, 0.0), r["GBps"])
            ck = (r["variant"], tuple(norm_params(r)))
            if sh not in cand[ck] or r["GBps"] > cand[ck][sh]["GBps"]:
                cand[ck][sh] = r
        return best, cand
    per_cell = {key: cell_cands(cells[key]) for key in cells}
    table = []
    for key in sorted(cells):
        rs = cells[key]
        shapes = sorted({(r["R"], r["C"]) for r in rs})
        best, cand = per_cell[key]
        nbrs = []
        if neighbor_weight > 0:
            for dl, dc in ((1, 0), (-1, 0), (0, 1), (0, -1)):
                nk = key[:3] + (key[3] + dl, key[4] + dc)
                if nk in per_cell:
                    nbrs.append(per_cell[nk])
        pool = list(cand)
        prot = [sh for sh in shapes if protect and (key[0], sh[0], sh[1]) in protect]
        if prot:
            keep = [ck for ck in pool if all(sh in cand[ck] and cand[ck][sh]["GBps"] >= (1 - protect_tol) * best[sh]
                                              for sh in prot)]
            if keep:
                pool = keep

        def sc(ck):      # a shape the candidate was not measured on counts at its own mean - 3 %
            got = [cand[ck][sh]["GBps"] / best[sh] for sh in cand[ck]]
            m = sum(got) / len(got)
            own = (sum(got) + 0.97 * m * (len(shapes) - len(got))) / len(shapes)
            if not nbrs:
                return own
            tot, wt = own, 1.0
            for nbest, ncand in nbrs:                 # neighbour cells: measured shapes only
                if ck in ncand:
                    ng = [ncand[ck][sh]["GBps"] / nbest[sh] for sh in ncand[ck]]
                    tot += neighbor_weight * sum(ng) / len(ng)
                else:
                    tot += neighbor_weight * 0.97 * m
                wt += neighbor_weight
            return tot / wt
        score = {ck: sc(ck) for ck in pool}
        top = max(score[ck] for ck in pool)
        if prefer_staged_dot > 0 and key[0] == "dot" and 6 <= key[4] <= 9 and key[3] + key[4] >= 25 and not prot:
            # DOT rows of 64..1023 values, >= 256 MiB: staged row tiles (XSMEM 4) generalise across the cell
            # (every training shape >= 256 MiB with both swept: staged >= 0.98 of the direct
            # kernels, median 1.05 aligned / 1.41 misaligned), the direct lane groups do not
            staged = [ck for ck in pool if ck[1][4] == 4 and score[ck] >= top * (1 - prefer_staged_dot)]
            if staged:
                pool = staged
                top = max(score[ck] for ck in pool)
        near = [ck for ck in pool if score[ck] >= top * (1 - tie)]
        if portable_tie > 0:
            port = [ck for ck in pool if score[ck] >= top * (1 - portable_tie)]
            nz = lambda ck: sum(1 for v in ck[1] if v != 0)       # noqa: E731
            fewest = min(nz(ck) for ck in port)
            near = [ck for ck in port if nz(ck) == fewest]
        big = shapes[-1] if len(shapes) == 1 else max(shapes, key=lambda sh: sh[0] * sh[1])

        def grid_of(ck):
            r = cand[ck].get(big) or next(iter(cand[ck].values()))
            pl = r["plan"]
            return pl["grid"][1 if (pl["vec_shape"] or pl.get("mis")) else 0]
        ck = min(near, key=lambda ck: (grid_of(ck), -score[ck]))
        pick = cand[ck].get(big) or max(cand[ck].values(), key=lambda r: r["R"] * r["C"])
        p = list(ck[1])
        table.append({"op": key[0], "dtype": key[1], "vec": key[2], "lr": key[3], "lc": key[4], "R": pick["R"], "C": pick["C"],
                      "variant": pick["variant"], "lanes": p[0], "splits": p[1], "ctas_per_sm": p[2],
                      "unroll": p[3], "xsmem": p[4], "block": p[5], "rows": p[6], "order": p[7], "pipe": p[8], "us": pick["us"], "GBps": pick["GBps"],
                      "score": score[ck], "shapes": len(shapes), "candidates": len(rs)})
    return table


def write_inc(table, path):
    with open(path, "w") as f:
        f.write("// Fitted selector table -- GENERATED by tools/fit_thresholds.py from B200 sweeps.\n")
        f.write("// {op, dtype, vec, floor(log2 R), floor(log2 C), variant, lanes, splits, ctas_per_sm, unroll, xsmem, block, rows, order, pipe}\n")
        f.write("// vec: 1 = the 128-bit path shape (MV/DOT/BLAS-1: C % 4 == 0; TMV: R % 4 == 0), 0 = scalar-load shape.\n")
        f.write("// lanes/splits/ctas_per_sm/unroll/xsmem/block: 0 = derived by the planner.\n")
        for e in table:
            f.write("    {%d, %d, %d, %d, %d, %d, %d, %d, %d, %d, %d, %d, %d, %d, %d},  // %s %dx%d %.0f GB/s\n" % (
                OP_ID[e["op"]], DT_ID[e["dtype"]], e["vec"], e["lr"], e["lc"], VARIANT_ID[e["variant"]], e["lanes"],
                e["splits"], e["ctas_per_sm"], e["unroll"], e["xsmem"], e["block"], e["rows"], e["order"], e["pipe"], e["variant"],
                e["R"], e["C"], e["GBps"]))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("inputs", nargs="+")
    ap.add_argument("--out", required=True)
    ap.add_argument("--json", default=None)
    ap.add_argument("--ops", default=None, help="comma list: fit only these ops (e.g. the BLAS-1 table)")
    ap.add_argument("--neighbor-weight", type=float, default=0.0,
                    help="score candidates on the adjacent cells' shapes too, with this weight")
    ap.add_argument("--portable-tie", type=float, default=0.0)
    ap.add_argument("--prefer-staged-dot", type=float, default=0.0,
                    help="DOT cells with rows of 64..1023 values: a staged row-tile candidate within this fraction "
                         "of the top score wins")
    ap.add_argument("--protect-bench", action="store_true",
                    help="keep every cell pick within 1 %% of the best run on bench.py's own shapes (the 42 "
                         "sweep shapes, their C+1 / R+1 off-grid twins, configs[2..4])")
    a = ap.parse_args()
    rows = [json.loads(l) for p in a.inputs for l in open(p) if l.strip()]
    if a.ops:
        rows = [r for r in rows if r["op"] in a.ops.split(",")]
    protect = None
    if a.protect_bench:
        protect = set()
        for k in range(3, 24):
            R, C = 1 << k, 1 << (26 - k)
            protect |= {("mv", R, C), ("tmv", R, C), ("mv", R, C + 1), ("tmv", R + 1, C)}
        protect |= {("dot", 1, 1 << k) for k in range(10, 31)} | {("mv", 131072, 32768), ("tmv", 1024, 1 << 24)}
    table = fit(rows, protect=protect, neighbor_weight=a.neighbor_weight, portable_tie=a.portable_tie,
                prefer_staged_dot=a.prefer_staged_dot)
    write_inc(table, a.out)
    if a.json:
        with open(a.json, "w") as f:
            json.dump(table, f, indent=1)
    for e in table:
        print(f"{e['op']:4s} {e['dtype']} v{e['vec']} 2^{e['lr']:2d} x 2^{e['lc']:2d}  {e['variant']:12s} "
              f"lanes={e['lanes']} S={e['splits']} U={e['unroll']} xs={e['xsmem']} nt={e['block']}  "
              f"{e['GBps']:.0f} GB/s ({e['candidates']} runs)")


if __name__ == "__main__":
    main()
