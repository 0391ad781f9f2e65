#!/usr/bin/env python
"""Merge the DRAM bytes of an `ncu --set full` capture of one bench step into
profiles/ncu_traffic.json (the bench's roofline.traffic lookup), keyed like
bench.Problem.key(): "<op>[x<K>]:<R>x<C>:<VARIANT>".

  python tools/merge_traffic.py gpurun_out/full_stencil_r1c_raw.csv gpurun_out/detail_stencil_r1c.jsonl
The capture must list the step's kernels in the bench's problem order (tools/profile_workload.sh).
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_summary import read  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main():
    raw, detail = sys.argv[1], sys.argv[2]
    out = sys.argv[3] if len(sys.argv) > 3 else os.path.join(ROOT, "profiles", "ncu_traffic.json")
    rows = read(raw)
    probs = [json.loads(l) for l in open(detail)]
    if len(rows) < len(probs):
        sys.exit(f"capture has {len(rows)} kernels, the step {len(probs)}")
    tr = json.load(open(out)) if os.path.exists(out) else {}
    for r, p in zip(rows, probs):
        k = p["plan"].get("nvec", 1)
        key = f"{p['op']}{'' if k == 1 else 'x%d' % k}:{p['R']}x{p['C']}:{p['variant']}"
        if "dram_bytes" in r:
            tr[key] = r["dram_bytes"]
            print(key, r["dram_bytes"], r["kernel"][:40])
    json.dump(tr, open(out, "w"), indent=1)


if __name__ == "__main__":
    main()
