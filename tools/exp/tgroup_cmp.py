#!/usr/bin/env python
"""Round-2 experiment: the four-row-group TMV kernel (XSMEM 12) against the selector's pick on
the offgrid bench's R + 1 TMV shapes (256 MiB).  Per candidate: median of 15 single launches
(CUDA events on the launching stream; the 256 MiB matrix is 2x L2).  JSONL to stdout."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_pldi_samadihmlm12_b200 as adaptic  # noqa: E402
from paper_conf_pldi_samadihmlm12_b200 import _lib as L  # noqa: E402


def timeit(plan, M, X, y, s, reps=15):
    ts = []
    for _ in range(3):
        plan.run(M.data_ptr(), X.data_ptr(), y.data_ptr(), s)
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        plan.run(M.data_ptr(), X.data_ptr(), y.data_ptr(), s)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    return statistics.median(ts)


def main():
    dev = torch.device("cuda:0")
    s = torch.cuda.current_stream().cuda_stream
    shapes = [((1 << k) + 1, 1 << (26 - k)) for k in range(2, 13)] + [(5, 13421772), (63, 1 << 20), (1537, 43690)]
    if len(sys.argv) > 1:
        shapes = [tuple(int(v) for v in t.split("x")) for t in sys.argv[1].split(",")]
    for R, C in shapes:
        M = torch.empty(R * C, dtype=torch.float32, device=dev)
        synth.device_matrix(M, R, C, "tmv", "uniform", 1)
        X = torch.empty(C, dtype=torch.float32, device=dev)
        synth.device_vector(X, "uniform", 2)
        y = torch.empty(R, dtype=torch.float32, device=dev)
        nb = 4 * (R * C + R + C)
        cands = [("AUTO", None)]
        for S in (1, 2, 3, 4):
            for U in (0, 8, 2):
                for order in (1, 2):
                    for nt in (0, 256, 512, 1024):
                        cands.append(("TMV_SPLITK", [0, 0, 0, U, 12, nt, S, order, 0]))
        for v, p in cands:
            try:
                plan = adaptic.get_plan(L.OP_TMV, R, C, L.F32, dev, v, p, s)
            except Exception:  # noqa: BLE001
                continue
            d = plan.describe()
            us = timeit(plan, M, X, y, s)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(20):
                plan.run(M.data_ptr(), X.data_ptr(), y.data_ptr(), s)
            e1.record()
            torch.cuda.synchronize()
            us_b2b = e0.elapsed_time(e1) * 1e3 / 20
            print(json.dumps({"R": R, "C": C, "variant": d["variant"], "params": p, "xmode": d["xmode"],
                              "block": d["block"], "S": d["rows_per_group"], "U": d["unroll"],
                              "grid": d["grid"], "us": us, "GBps": nb / us / 1e3, "us_b2b": us_b2b,
                              "GBps_b2b": nb / us_b2b / 1e3}), flush=True)
        del M, X, y


if __name__ == "__main__":
    main()
