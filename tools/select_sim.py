#!/usr/bin/env python
"""Offline replica of the selector's table lookup (csrc/adaptic.cu table_lookup_scan) to
predict, from a fitted table (tools/fit_thresholds.py --json) and a full-grid sweep of some
shapes (tools/sweep.py), what AUTO would run on each shape and how fast that candidate
measured there -- so a fitting rule can be judged on held-out shapes without a GPU run.

Prediction = the measured GB/s of the sweep candidate whose (variant, portable params)
equals the looked-up cell entry; shapes whose entry was not among the swept candidates
(a projected cell with re-derived splits, or the heuristic fallback) are 'unpredicted'.

  python tools/select_sim.py --table profiles/selector_table_r2.json gpurun_out/r2_heldoutB.jsonl
"""
import argparse
import collections
import gzip
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from fit_thresholds import norm_params  # noqa: E402

BEYOND_L2_LOG2 = 26


def lookup(table, op, dtype, R, C):
    """Port of table_lookup_scan: nearest cell (Manhattan <= 2, ties: closer element count,
    then table order), else projection onto the largest measured diagonal >= 2^26 at the same
    aspect (splits / CTAs re-derived), else int32 -> fp32.  Returns (entry, projected)."""
    lr, lc = R.bit_length() - 1, C.bit_length() - 1
    vec = int((R % 4 == 0) if op == "tmv" else (C % 4 == 0))
    best, bestd = None, 1 << 30
    for e in table:
        if e["op"] != op or e["dtype"] != dtype or e["vec"] != vec:
            continue
        d = abs(e["lr"] - lr) + abs(e["lc"] - lc)
        if d < bestd or (d == bestd and best is not None and
                         abs(e["lr"] + e["lc"] - lr - lc) < abs(best["lr"] + best["lc"] - lr - lc)):
            best, bestd = e, d
    if best is not None and bestd <= 2:
        return best, False
    diag = max([e["lr"] + e["lc"] for e in table if e["op"] == op and e["dtype"] == dtype and e["vec"] == vec
                and e["lr"] + e["lc"] <= lr + lc] or [-1])
    if diag >= BEYOND_L2_LOG2:
        pb, pd = None, 1 << 30
        for e in table:
            if e["op"] != op or e["dtype"] != dtype or e["vec"] != vec or e["lr"] + e["lc"] != diag:
                continue
            d = abs((e["lr"] - e["lc"]) - (lr - lc))
            if d < pd:
                pb, pd = e, d
        if pb is not None and pd <= 2:
            return pb, True
    if dtype != "f32":
        return lookup(table, op, "f32", R, C)
    return None, False


def entry_key(e):
    return (e["variant"], (e["lanes"], e["splits"], e["ctas_per_sm"], e["unroll"], e["xsmem"], e["block"],
                           e["rows"], e["order"], e["pipe"]))


def load(paths):
    out = []
    for p in paths:
        op = gzip.open if p.endswith(".gz") else open
        with op(p, "rt") as f:
            out += [json.loads(l) for l in f if l.strip()]
    return out


def evaluate(table, rows, min_bytes=256 * 2 ** 20, peak=6554.9):
    """Per shape: (op, R, C, predicted GB/s or None, best fixed GB/s, measured AUTO GB/s or None)."""
    shapes = collections.defaultdict(dict)
    auto = {}
    for r in rows:
        key = (r["op"], r["dtype"], r["R"], r["C"])
        if r["req"] == "AUTO":
            auto[key] = r["GBps"]
            continue
        ck = (r["variant"], tuple(norm_params(r)))
        shapes[key][ck] = max(shapes[key].get(ck, 0.0), r["GBps"])
    out = []
    for key, cands in sorted(shapes.items()):
        op, dt, R, C = key
        nb = 4 * (R * C * (2 if op == "dot" else 1) + R + (0 if op == "dot" else C))
        if nb < min_bytes:
            continue
        e, proj = lookup(table, op, dt, R, C)
        pred = None
        if e is not None and not proj:
            pred = cands.get(entry_key(e))
        out.append({"op": op, "dtype": dt, "R": R, "C": C, "pred": pred, "best": max(cands.values()),
                     "auto": auto.get(key), "entry": e and entry_key(e), "projected": proj})
    return out


def summarise(res, peak=6554.9, tol=0.95):
    n = len(res)
    pred = [r for r in res if r["pred"] is not None]
    ok = [r for r in pred if r["pred"] >= tol * r["best"] and r["pred"] >= 0.7 * peak]
    return {"shapes": n, "predicted": len(pred), "pass": len(ok)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("sweeps", nargs="+")
    ap.add_argument("--table", required=True)
    a = ap.parse_args()
    table = json.load(open(a.table))
    res = evaluate(table, load(a.sweeps))
    print(json.dumps(summarise(res)))
    for r in res:
        if r["pred"] is None or r["pred"] < 0.95 * r["best"]:
            print(r["op"], r["R"], r["C"], "pred", r["pred"] and round(r["pred"]), "best", round(r["best"]),
                  "auto", r["auto"] and round(r["auto"]), r["entry"], "proj" if r["projected"] else "")


if __name__ == "__main__":
    main()
