#!/usr/bin/env python
"""Summarise ncu reports (.ncu-rep) into JSON / markdown for profiles/.

  python tools/ncu_summary.py gpurun_out/bench_full.ncu-rep --keys bench_keys.json \
      --json profiles/r1_ncu_bench.json --md profiles/r1_ncu_bench.md --traffic profiles/ncu_traffic.json

--keys: optional JSON list naming each captured launch in order (e.g. the bench's
problem keys "op:RxC:VARIANT"); --traffic writes {key: dram_read+write bytes}
(bench.py reports it as roofline.traffic).
"""
import argparse
import csv
import io
import json
import subprocess

METRICS = {
    "gpu__time_duration.sum": "duration",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct2",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "achieved_occupancy_pct",
    "launch__registers_per_thread": "registers",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
    "launch__occupancy_limit_registers": "occ_limit_regs",
    "lts__t_sectors_srcunit_tex_op_read.sum": "l2_read_sectors",
    "smsp__average_warp_latency_issue_stalled_long_scoreboard.ratio": "stall_long_sb",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio": "stall_long_sb_per_issue",
    "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio": "stall_barrier_per_issue",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_pct",
}
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1,
         "msecond": 1e-3, "second": 1}


def read(rep):
    if rep.endswith(".csv"):              # an exported raw page (ncu -i X --page raw --csv)
        out = open(rep).read()
    else:
        out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    head, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[head.index("Kernel Name")] if "Kernel Name" in head else ""}
        for m, name in METRICS.items():
            if m in head:
                i = head.index(m)
                v = r[i].replace(",", "")
                try:
                    val = float(v) * SCALE.get(units[i], 1)
                except ValueError:
                    continue
                d[name] = val
        if "dram_read" in d and "dram_write" in d:
            d["dram_bytes"] = d["dram_read"] + d["dram_write"]
            if d.get("duration"):
                d["dram_GBps"] = d["dram_bytes"] / d["duration"] / 1e9
        res.append(d)
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("reps", nargs="+")
    ap.add_argument("--keys", default=None)
    ap.add_argument("--json", default=None)
    ap.add_argument("--md", default=None)
    ap.add_argument("--traffic", default=None)
    ap.add_argument("--detail", default=None,
                    help="bench.py --detail JSONL of the captured step: keys op:RxC:VARIANT in launch order; a "
                         "plan's pre-kernel (x_shift_kernel) is folded into the next problem's DRAM bytes")
    a = ap.parse_args()
    rows = [r for rep in a.reps for r in read(rep)]
    keys = json.load(open(a.keys)) if a.keys else [None] * len(rows)
    if a.detail:
        det = [json.loads(l) for l in open(a.detail) if l.strip()]
        dk = iter(f"{q['op']}:{q['R']}x{q['C']}:{q['variant']}" for q in det)
        keys, extra = [], 0.0
        for r in rows:
            if "x_shift" in r["kernel"]:
                keys.append(None)
                extra += r.get("dram_bytes", 0.0)
                continue
            keys.append(next(dk, None))
            if extra and "dram_bytes" in r:
                r["dram_bytes"] += extra
                r["prekernel_bytes"] = extra
            extra = 0.0
    for r, k in zip(rows, keys):
        r["key"] = k
    if a.json:
        json.dump(rows, open(a.json, "w"), indent=1)
    if a.traffic:
        json.dump({r["key"]: r["dram_bytes"] for r in rows if r.get("key") and "dram_bytes" in r},
                  open(a.traffic, "w"), indent=1)
    lines = ["| launch | kernel | us | DRAM MB (r+w) | DRAM GB/s | regs | occ % | grid |", "|---|---|---|---|---|---|---|---|"]
    for r in rows:
        lines.append("| %s | %s | %.1f | %.1f | %.0f | %s | %.0f | %s |" % (
            r.get("key") or "", r["kernel"][:60], r.get("duration", 0) * 1e6, r.get("dram_bytes", 0) / 1e6,
            r.get("dram_GBps", 0), int(r.get("registers", 0)), r.get("achieved_occupancy_pct", 0),
            int(r.get("grid", 0))))
    text = "\n".join(lines)
    if a.md:
        open(a.md, "w").write(text + "\n")
    print(text)


if __name__ == "__main__":
    main()
