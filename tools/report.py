#!/usr/bin/env python
"""Selector report from a sweep (tools/sweep.py JSONL): per shape the AUTO pick, the
best fixed (variant, params), their ratio, and the fraction of the HBM peak -- the
BJ:north_star gates ("the selector's chosen variant reaches >= 70 % of B200 HBM
bandwidth ... for inputs >= 256 MB and is within 5 % of the best hand-picked
variant for that shape").

  python tools/report.py profiles/sweep_*.jsonl --peak 6546.9 --md profiles/r1_selector_report.md
"""
import argparse
import collections
import json
import os


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("inputs", nargs="+")
    ap.add_argument("--peak", type=float, default=None, help="HBM GB/s (default MEASURED_PEAKS.json)")
    ap.add_argument("--md", default=None)
    ap.add_argument("--min-bytes", type=float, default=256 * 2 ** 20, help="gate applies at >= this many bytes")
    ap.add_argument("--no-peak-gate", action="store_true",
                    help="small (L2-resident) shapes: gate only on AUTO >= 0.95 x best fixed")
    ap.add_argument("--best-from", nargs="*", default=[],
                    help="sweeps whose fixed-variant runs give 'best fixed' (AUTO is taken from the inputs)")
    a = ap.parse_args()
    peak = a.peak
    if peak is None:
        p = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")
        peak = json.load(open(p))["hbm_gbs"] if os.path.exists(p) else 6650.0
    import gzip

    def load(paths):
        out = []
        for path in paths:
            op = gzip.open if path.endswith(".gz") else open
            with op(path, "rt") as f:
                out += [json.loads(l) for l in f if l.strip()]
        return out
    rows = load(a.inputs)
    if a.best_from:
        rows = [r for r in rows if r["req"] == "AUTO"] + [r for r in load(a.best_from) if r["req"] != "AUTO"]
    by = collections.defaultdict(list)
    for r in rows:
        by[(r["op"], r["dtype"], r["R"], r["C"])].append(r)
    out = ["| op | R x C | bytes | AUTO variant | AUTO GB/s | best fixed | best GB/s | AUTO/best | AUTO/peak | gates |",
           "|---|---|---|---|---|---|---|---|---|---|"]
    n_gate = n_pass = n_10 = n_peak = 0
    worst = []
    for key in sorted(by, key=lambda k: (k[0], k[1], k[2] * k[3], k[2])):
        rs = by[key]
        auto = [r for r in rs if r["req"] == "AUTO"]
        fixed = [r for r in rs if r["req"] != "AUTO"]
        if not auto or not fixed:
            continue
        au = min(auto, key=lambda r: r["us"])
        be = min(fixed, key=lambda r: r["us"])
        opn, dt, R, C = key
        nbytes = au["GBps"] * au["us"] * 1e3
        ratio = be["us"] / au["us"]
        frac = au["GBps"] / peak
        gate = ""
        if nbytes >= a.min_bytes:
            ok = ratio >= 0.95 and (a.no_peak_gate or frac >= 0.70)
            n_gate += 1
            n_pass += ok
            n_10 += ratio >= 0.90
            n_peak += frac >= 0.70
            gate = "PASS" if ok else "FAIL"
            worst.append((ratio, f"{opn} {R}x{C}"))
        out.append(f"| {opn} {dt} | {R}x{C} | {nbytes / 2**20:.0f} MiB | {au['variant']} | {au['GBps']:.0f} | "
                   f"{be['variant']} {be['params']} | {be['GBps']:.0f} | {ratio:.3f} | {frac:.3f} | {gate} |")
    out.append("")
    gate_txt = "AUTO >= 0.95 x best fixed" + ("" if a.no_peak_gate else " and >= 0.70 x peak")
    out.append(f"peak = {peak:.1f} GB/s; gated shapes (>= {a.min_bytes / 2**20:.0f} MiB): {n_pass}/{n_gate} pass "
               f"({gate_txt}); {n_10}/{n_gate} within 10 % of the best fixed; {n_peak}/{n_gate} >= 0.70 of peak.")
    if worst:
        worst.sort()
        out.append("lowest AUTO/best: " + ", ".join(f"{w[1]} {w[0]:.3f}" for w in worst[:5]))
    text = "\n".join(out)
    if a.md:
        open(a.md, "w").write(text + "\n")
    print(text)


if __name__ == "__main__":
    main()
