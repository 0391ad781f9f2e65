#!/usr/bin/env python
"""Time AUTO and given forced candidates on given shapes (round-2 experiments): median of 15
single launches and the mean of 20 back-to-back launches (CUDA events on the launching stream).

  python tools/exp/cand_cmp.py tmv 513x131072,129x524288 "TMV_REGTILE:0,0,2,0,4,544,0" ...
JSONL to stdout."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_pldi_samadihmlm12_b200 as adaptic  # noqa: E402
from paper_conf_pldi_samadihmlm12_b200 import _lib as L  # noqa: E402


def times(plan, M, X, y, s, reps=15):
    for _ in range(3):
        plan.run(M.data_ptr(), X.data_ptr(), y.data_ptr(), s)
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        plan.run(M.data_ptr(), X.data_ptr(), y.data_ptr(), s)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(20):
        plan.run(M.data_ptr(), X.data_ptr(), y.data_ptr(), s)
    e1.record()
    torch.cuda.synchronize()
    return statistics.median(ts), e0.elapsed_time(e1) * 1e3 / 20


def main():
    op = sys.argv[1]
    shapes = [tuple(int(v) for v in t.split("x")) for t in sys.argv[2].split(",")]
    cands = [("AUTO", None)]
    for c in sys.argv[3:]:
        v, p = c.split(":")
        cands.append((v, [int(t) for t in p.split(",")] + [0] * 9))
    dev = torch.device("cuda:0")
    s = torch.cuda.current_stream().cuda_stream
    for R, C in shapes:
        M = torch.empty(R * C, dtype=torch.float32, device=dev)
        synth.device_matrix(M, R, C, "tmv" if op == "tmv" else "mv", "uniform", 1)
        X = torch.empty(C, dtype=torch.float32, device=dev)
        synth.device_vector(X, "uniform", 2)
        y = torch.empty(R, dtype=torch.float32, device=dev)
        nb = 4 * (R * C + R + C)
        for v, p in cands:
            try:
                plan = adaptic.get_plan(L.OPS[op], R, C, L.F32, dev, v, p[:9] if p else None, s)
            except Exception as e:  # noqa: BLE001
                print(json.dumps({"R": R, "C": C, "variant": v, "params": p and p[:9], "error": str(e)[:80]}))
                continue
            d = plan.describe()
            us, us_b2b = times(plan, M, X, y, s)
            print(json.dumps({"R": R, "C": C, "variant": d["variant"], "params": p and p[:9], "plan": d, "us": us,
                              "GBps": nb / us / 1e3, "us_b2b": us_b2b, "GBps_b2b": nb / us_b2b / 1e3}), flush=True)
        del M, X, y


if __name__ == "__main__":
    main()
