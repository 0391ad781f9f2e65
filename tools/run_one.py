#!/usr/bin/env python
"""Run one (op, R, C, variant[, params]) problem `reps` times -- a target for ncu.

  python tools/run_one.py tmv 8388608 8 TMV_COL --reps 3 [--params 256,1,4,8]
Prints the plan and the CUDA-event time per launch (median).
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_pldi_samadihmlm12_b200 as adaptic  # noqa: E402
from paper_conf_pldi_samadihmlm12_b200 import _lib as L  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("op")
    ap.add_argument("R", type=int)
    ap.add_argument("C", type=int)
    ap.add_argument("variant", nargs="?", default="AUTO")
    ap.add_argument("--params", default=None)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--dtype", default="f32")
    a = ap.parse_args()
    params = [int(v) for v in a.params.split(",")] if a.params else None
    tdt = torch.float32 if a.dtype == "f32" else torch.int32
    dev = torch.device("cuda:0")
    M = torch.empty(a.R * a.C, dtype=tdt, device=dev)
    synth.device_matrix(M, a.R, a.C, "tmv" if a.op == "tmv" else "mv", "uniform", 1)
    X = torch.empty(a.R * a.C if a.op == "dot" else a.C, dtype=tdt, device=dev)
    if a.op == "dot":
        synth.device_matrix(X, a.R, a.C, "mv", "uniform", 2)
    else:
        synth.device_vector(X, "uniform", 2)
    y = torch.empty(a.R, dtype=tdt, device=dev)
    opc = {"mv": L.OP_MV, "tmv": L.OP_TMV, "dot": L.OP_DOT}[a.op]
    s = torch.cuda.current_stream().cuda_stream
    plan = adaptic.get_plan(opc, a.R, a.C, L.F32 if a.dtype == "f32" else L.I32, dev, a.variant, params, s)
    print(json.dumps(plan.describe()))
    ts = []
    for _ in range(a.reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        plan.run(M.data_ptr(), X.data_ptr(), y.data_ptr(), s)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    nbytes = 4 * (a.R * a.C * (2 if a.op == "dot" else 1) + a.R + (0 if a.op == "dot" else a.C))
    med = statistics.median(ts)
    print(json.dumps({"us_median": med, "GBps": nbytes / med / 1e3, "all_us": ts}))


if __name__ == "__main__":
    main()
