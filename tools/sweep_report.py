#!/usr/bin/env python
"""Summarise a sweep JSONL: per shape the AUTO pick, the best run and the best per variant."""
import collections
import json
import sys


def main(paths):
    rows = [json.loads(l) for p in paths for l in open(p)]
    by = collections.defaultdict(list)
    for r in rows:
        by[(r["op"], r["dtype"], r["R"], r["C"])].append(r)
    for key in sorted(by, key=lambda k: (k[0], k[1], k[2])):
        rs = sorted(by[key], key=lambda r: r["us"])
        auto = [r for r in rs if r["req"] == "AUTO"]
        pv = {}
        for r in rs:
            pv.setdefault(r["variant"], r)
        s = " ".join(f"{v[:10]}:{pv[v]['GBps']:.0f}" for v in sorted(pv, key=lambda v: -pv[v]["GBps"]))
        a = f"AUTO {auto[0]['variant']} {auto[0]['GBps']:.0f}" if auto else "AUTO -"
        print(key, a, f"| best {rs[0]['variant']} {rs[0]['params']} {rs[0]['GBps']:.0f} |", s)


if __name__ == "__main__":
    main(sys.argv[1:])
