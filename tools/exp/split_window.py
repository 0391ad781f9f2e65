#!/usr/bin/env python
"""Experiment: does a compact DRAM address window help?  MV_SPLIT with growing split
counts S (contiguous chunks, order 1, vs interleaved, order 2) on shapes where every
row is its own stream.  Prints GB/s per (shape, S, order)."""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_pldi_samadihmlm12_b200 as adaptic  # noqa: E402
from paper_conf_pldi_samadihmlm12_b200 import _lib as L  # noqa: E402
from tools.sweep import time_plan  # noqa: E402

dev = torch.device("cuda:0")
stream = torch.cuda.current_stream().cuda_stream
for R, C in [(1024, 65536), (4096, 16384), (64, 1 << 20), (8192, 8192), (256, 262144)]:
    M = torch.empty(R * C, dtype=torch.float32, device=dev)
    synth.device_matrix(M, R, C, "mv", "uniform", 1)
    X = torch.empty(C, dtype=torch.float32, device=dev)
    synth.device_vector(X, "uniform", 2)
    Y = torch.empty(R, dtype=torch.float32, device=dev)
    ptrs = (M.data_ptr(), X.data_ptr(), Y.data_ptr())
    nbytes = 4 * (R * C + R + C)
    for v, p in [("AUTO", None), ("MV_CPR", [256, 0, 0, 4]), ("MV_CPR", [256, 0, 0, 4, 0, 0, 2])]:
        plan = adaptic.get_plan(L.OP_MV, R, C, L.F32, dev, v, p, stream)
        us = statistics.median(time_plan(plan, ptrs, stream, 7))
        print(f"{R}x{C} {v} {p} {plan.describe()['variant']} {nbytes / us / 1e3:.0f} GB/s", flush=True)
    for S in (2, 4, 8, 16, 32, 64, 128):
        for order in (1, 2):
            for rb, u in ((1, 4), (2, 2)):
                try:
                    plan = adaptic.get_plan(L.OP_MV, R, C, L.F32, dev, "MV_SPLIT", [256, S, 0, u, 0, 0, rb, order], stream)
                except adaptic.AdapticError:
                    continue
                us = statistics.median(time_plan(plan, ptrs, stream, 7))
                print(f"{R}x{C} SPLIT S={S} order={order} rb={rb} u={u} grid={plan.describe()['grid'][1]} "
                      f"{nbytes / us / 1e3:.0f} GB/s", flush=True)
    adaptic.clear_cache()
    del M
