#!/usr/bin/env python
"""Analytic performance model of the variants -- the paper's
selection mechanism, checked against the measured selector.

Adaptic's compiler picks kernels with "a high-level performance model ... that
classifies CUDA kernels into three categories of memory-bound, computation-bound,
and latency-bound": a kernel is latency-bound when "there are not enough
active warps on each SM" to hide memory latency; otherwise its time is the larger of
its memory and computation times; the break-even points between kernels give the
input subranges.  The B200 build measures instead (tools/sweep.py ->
tools/fit_thresholds.py); this tool states the model for B200 and asks how close its
choices come to the measured best.

Per plan (the planner's own description: grid, block, CTAs per SM, loads in flight):
  warps/SM  w = min(grid, sms*cps)/sms * block/32
  in flight F = w * 32 * loads_per_thread * 16 B             (Little's law)
  bandwidth BW = min(peak, sms * F / latency)                 (latency-bound below peak)
  t_mem     = bytes / BW  stretched by the last-wave imbalance ceil(n/g)/(n/g)
  t_comp    = elements * ops_per_element / (sms * 4 warps-issue/clk * 32 * clock)
  t         = t0 + max(t_mem, t_comp) (+ per-work-item overhead x items per CTA, and a
              merge term when a reduction is split across CTAs)
Free constants (latency, t0, overheads) are fitted on the fixed-variant sweeps by least
squares in log time; the report compares, per shape, the measured time of the model's
pick with the measured best and with the table-driven selector's pick.

  python tools/perf_model.py profiles/sweep_r1_main_fit.jsonl.gz --md profiles/r1_perf_model.md
"""
import argparse
import collections
import gzip
import json
import math

import numpy as np
from scipy.optimize import least_squares

SMS = 148
CLOCK = 1.9e9
PEAK = 7.2e12                      # steady read bandwidth of the 16-64 GiB shapes (profiles/)


def load(paths):
    rows = []
    for p in paths:
        op = gzip.open if p.endswith(".gz") else open
        with op(p, "rt") as f:
            rows += [json.loads(l) for l in f if l.strip()]
    return rows


def features(r):
    """(bytes, warps/SM, loads in flight per thread, items, grid, has_merge, kind, elems)."""
    d = r["plan"]
    w = 1 if (d["vec_shape"] or d.get("mis")) else 0
    grid = max(1, d["grid"][w])
    cps = max(1, d["ctas_per_sm"])
    block = max(32, d["block"])
    R, C, v = r["R"], r["C"], d["variant"]
    U, RB, S = max(1, d["unroll"]), max(1, d["rows_per_group"]), max(1, d["splits"])
    width = 16 if w else 4
    if v == "MV_TPR":
        loads, items, kind = 8 * d.get("stages", 2), math.ceil(R / d["lanes"]), "tpr"
        width = 16
    elif v in ("MV_SUBWARP", "MV_WPR"):
        G = max(1, d["lanes"])
        loads, items, kind = U * RB, math.ceil(R / (RB * 32 // G)), "group"
    elif v in ("MV_CPR", "MV_SPLIT"):
        loads, items, kind = U * RB, math.ceil(R / RB) * S, "cta"
    else:
        LR = max(1, d["lanes"])
        rv = R // 4 if d["vec_shape"] else R
        loads, items, kind = U, math.ceil(rv / LR) * S, "tmv"
    resident = min(grid, SMS * cps) / SMS
    warps = resident * block / 32
    nbytes = r["GBps"] * r["us"] * 1e3
    return nbytes, warps, loads * width, items, grid, S > 1, kind, R * C


def model_time(th, f):
    lat, t0, o_cta, o_group, o_tmv, o_merge = th
    nbytes, warps, fl, items, grid, merge, kind, elems = f
    inflight = warps * 32 * fl
    bw = min(PEAK, SMS * inflight / (lat * 1e-6))
    per = items / grid
    tail = math.ceil(per) / per if per > 0 else 1.0
    t_mem = nbytes / bw * tail
    t_comp = elems * 2 / (SMS * 4 * 32 * CLOCK)
    over = {"cta": o_cta, "group": o_group, "tmv": o_tmv, "tpr": o_group}[kind] * math.ceil(per)
    return t0 * 1e-6 + max(t_mem, t_comp) + over * 1e-6 + (o_merge * 1e-6 if merge else 0.0)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("inputs", nargs="+")
    ap.add_argument("--md", default=None)
    a = ap.parse_args()
    # HBM regime only (the model's bandwidth term is HBM's): >= 2^24 elements = 64 MiB
    rows = [r for r in load(a.inputs) if r["req"] != "AUTO" and r["dtype"] == "f32" and r["R"] * r["C"] >= 1 << 24]
    feats = [features(r) for r in rows]
    meas = np.array([r["us"] * 1e-6 for r in rows])

    def resid(th):
        return np.array([math.log(model_time(th, f)) for f in feats]) - np.log(meas)

    th0 = np.array([1.0, 3.0, 0.2, 0.05, 0.1, 2.0])
    fit = least_squares(resid, th0, bounds=([0.1, 0, 0, 0, 0, 0], [10, 50, 20, 5, 20, 50]))
    th = fit.x
    err = np.exp(np.abs(resid(th)))
    by = collections.defaultdict(list)
    for r, f in zip(rows, feats):
        by[(r["op"], r["R"], r["C"])].append((r, model_time(th, f)))
    out = [f"fitted: latency {th[0]:.2f} us, t0 {th[1]:.2f} us, per-item overhead cta {th[2]:.3f} / group "
           f"{th[3]:.3f} / tmv {th[4]:.3f} us, split merge {th[5]:.2f} us; median |model/measured| "
           f"{np.median(err):.3f}, p90 {np.percentile(err, 90):.3f} over {len(rows)} runs", "",
           "| op | R x C | measured best | model's pick | its measured time / best |", "|---|---|---|---|---|"]
    ratios = []
    for key in sorted(by, key=lambda k: (k[0], k[1] * k[2], k[1])):
        cands = by[key]
        best = min(cands, key=lambda c: c[0]["us"])
        pick = min(cands, key=lambda c: c[1])
        ratio = pick[0]["us"] / best[0]["us"]
        ratios.append(ratio)
        if key[1] * key[2] >= 1 << 24:
            out.append(f"| {key[0]} | {key[1]}x{key[2]} | {best[0]['variant']} {best[0]['us']:.1f} us | "
                       f"{pick[0]['variant']} {pick[0]['params']} | {ratio:.3f} |")
    ratios = np.array(ratios)
    out.insert(1, f"model's pick vs measured best over {len(ratios)} shapes: median slowdown {np.median(ratios):.3f}, "
                  f"within 5 %: {np.mean(ratios <= 1.05) * 100:.0f} %, within 20 %: {np.mean(ratios <= 1.2) * 100:.0f} %, "
                  f"worst {ratios.max():.2f}x (the measured table is within 5 % by construction)")
    text = "\n".join(out)
    if a.md:
        open(a.md, "w").write(text + "\n")
    print("\n".join(out[:3]))


if __name__ == "__main__":
    main()
