#!/usr/bin/env python
"""Merge sweep JSONL files (plain or .gz) into one fit input, later files winning.

A run is keyed by (op, dtype, R, C, variant, params): a later file's run replaces an
earlier run with the same key (a kernel re-measured after a change).  A file given as
"+path" was a FULL re-sweep of its shapes: every earlier run of those shapes is dropped
(so all candidates of a shape come from the same box and day).  AUTO runs are kept only
from the last file that has them for the shape.

  python tools/merge_sweeps.py out.jsonl profiles/sweep_r1_main_fit.jsonl.gz \
      profiles/sweep_r1_mv_tile.jsonl.gz +profiles/sweep_r1f_offgrid.jsonl.gz \
      profiles/sweep_r1f_tmvrt.jsonl.gz +profiles/sweep_r1g_tmvmis.jsonl.gz
"""
import gzip
import json
import sys


def load(path):
    op = gzip.open if path.endswith(".gz") else open
    with op(path, "rt") as f:
        return [json.loads(l) for l in f if l.strip()]


def main():
    out, inputs = sys.argv[1], sys.argv[2:]
    runs = {}
    for arg in inputs:
        full = arg.startswith("+")
        rows = load(arg[1:] if full else arg)
        shapes = {(r["op"], r["dtype"], r["R"], r["C"]) for r in rows}
        if full:
            runs = {k: v for k, v in runs.items() if k[:4] not in shapes}
        for r in rows:
            key = (r["op"], r["dtype"], r["R"], r["C"], r["req"] if r["req"] == "AUTO" else r["variant"],
                   json.dumps(r["params"]))
            runs[key] = r
    with open(out, "w") as f:
        for r in runs.values():
            f.write(json.dumps(r) + "\n")
    print(f"{len(runs)} runs from {len(inputs)} files -> {out}", file=sys.stderr)


if __name__ == "__main__":
    main()
