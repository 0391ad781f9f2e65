#!/usr/bin/env python
"""Per-kernel share of a bench step from an ncu launch list (gpu__time_duration.sum,
--clock-control none; cold-cache, serialised launches), beside the bench's own
live per-kernel timing (--detail JSONL).  ncu's absolute times are not bench
values; the SHARE of the step is what must agree.

  python tools/launch_share.py profiles/r1_ncu_launches.csv --detail gpurun_out/detail_prof.jsonl \
      --per-step 42 --skip 126 --steps 2 --md profiles/r1_ncu_launches_summary.md
"""
import argparse
import csv
import io
import json


def launches(path):
    lines = open(path).read().splitlines()
    i = next(k for k, l in enumerate(lines) if l.startswith('"ID"'))
    out = []
    for r in csv.DictReader(io.StringIO("\n".join(lines[i:]))):
        if r["Metric Name"] != "gpu__time_duration.sum":
            continue
        scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}[r["Metric Unit"]]
        out.append((r["Kernel Name"], float(r["Metric Value"].replace(",", "")) * scale))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("csv")
    ap.add_argument("--detail", required=True)
    ap.add_argument("--per-step", type=int, required=True)
    ap.add_argument("--skip", type=int, default=0, help="launches before the timed steps (warm-up)")
    ap.add_argument("--steps", type=int, default=1)
    ap.add_argument("--md", default=None)
    a = ap.parse_args()
    L = launches(a.csv)
    det = [json.loads(l) for l in open(a.detail)]
    n = a.per_step
    us = [0.0] * n
    for s in range(a.steps):
        for i in range(n):
            us[i] += L[a.skip + s * n + i][1] / a.steps
    tot = sum(us)
    live_tot = sum(d["us"] for d in det)
    rows = ["| # | problem | variant | ncu us (cold) | ncu share | bench us (live) | bench share |",
            "|---|---|---|---|---|---|---|"]
    for i, d in enumerate(det):
        rows.append(f"| {i} | {d['op']} {d['R']}x{d['C']} | {d['variant']} | {us[i]:.1f} | {us[i] / tot:.4f} | "
                    f"{d['us']:.1f} | {d['us'] / live_tot:.4f} |")
    dom = max(range(n), key=lambda i: det[i]["us"])
    rows.append("")
    rows.append(f"step: ncu sum {tot:.1f} us over {n} launches (cold, serialised); bench kernel sum {live_tot:.1f} us. "
                f"Dominant kernel (bench): #{dom} {det[dom]['op']} {det[dom]['R']}x{det[dom]['C']} {det[dom]['variant']}: "
                f"share {det[dom]['us'] / live_tot:.4f} live vs {us[dom] / tot:.4f} under ncu.")
    text = "\n".join(rows)
    if a.md:
        open(a.md, "w").write(text + "\n")
    print(text)


if __name__ == "__main__":
    main()
