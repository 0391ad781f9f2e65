#!/usr/bin/env python
"""Round-2 experiment: the column-chunk staged MV kernel (XSMEM 13) against the selector's pick
on long misaligned MV rows (the offgrid bench's C + 1 shapes and held-out long rows, 256 MiB+).
Per candidate: median of 15 single launches and the mean of 20 back-to-back launches (CUDA
events on the launching stream).  JSONL to stdout."""
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
    dev = torch.device("cuda:0")
    s = torch.cuda.current_stream().cuda_stream
    shapes = [(1 << k, (1 << (26 - k)) + 1) for k in range(2, 13)]
    if len(sys.argv) > 1:
        shapes = [tuple(int(v) for v in t.split("x")) for t in sys.argv[1].split(",")]
    for R, C in shapes:
        M = torch.empty(R * C, dtype=torch.float32, device=dev)
        synth.device_matrix(M, R, C, "mv", "uniform", 1)
        X = torch.empty(C, dtype=torch.float32, device=dev)
        synth.device_vector(X, "uniform", 2)
        y = torch.empty(R, dtype=torch.float32, device=dev)
        nb = 4 * (R * C + R + C)
        cands = [("AUTO", None)]
        for MX, NT in ((16, 512), (8, 512), (36, 512), (16, 256), (36, 256)):
            for k in (0, 1, 2, 4):
                for st in (0, 4):
                    cands.append(("MV_SPLIT", [MX, 0, 0, st, 13, NT, k, 0, 0]))
        for v, p in cands:
            try:
                plan = adaptic.get_plan(L.OP_MV, R, C, L.F32, dev, v, p, s)
            except Exception:  # noqa: BLE001
                continue
            d = plan.describe()
            us, us_b2b = times(plan, M, X, y, s)
            print(json.dumps({"R": R, "C": C, "variant": d["variant"], "params": p, "xmode": d["xmode"],
                              "block": d["block"], "lanes": d["lanes"], "k": d["rows_per_group"],
                              "nch": d["splits"], "stages": d["stages"], "grid": d["grid"], "us": us,
                              "GBps": nb / us / 1e3, "us_b2b": us_b2b, "GBps_b2b": nb / us_b2b / 1e3}), flush=True)
        del M, X, y


if __name__ == "__main__":
    main()
