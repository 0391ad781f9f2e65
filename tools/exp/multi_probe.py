#!/usr/bin/env python
"""Experiment: multi-vector MV variants/params on the bench shapes (GB/s)."""
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
K = 4
for R, C in [(65536, 1024), (8192, 8192), (64, 1 << 20)]:
    M = torch.empty(R * C, device=dev)
    synth.device_matrix(M, R, C, "mv", "uniform", 1)
    X = torch.empty(K * C, device=dev)
    synth.device_vector(X, "uniform", 2)
    Y = torch.empty(K * R, device=dev)
    nbytes = 4 * (R * C + K * (R + C))
    for v, p in [("AUTO", None), ("MV_CPR", [0, 0, 0, 1, 1]), ("MV_CPR", [0, 0, 0, 1, 2]), ("MV_CPR", [0, 0, 0, 2, 1]),
                 ("MV_CPR", [0, 0, 0, 2, 2]), ("MV_SPLIT", [0, 2, 0, 2]), ("MV_SPLIT", [0, 4, 0, 2])]:
        try:
            plan = adaptic.get_plan(L.OP_MV, R, C, L.F32, dev, v, p, stream, K)
        except adaptic.AdapticError as e:
            print(R, C, v, p, "ERR", e)
            continue
        us = statistics.median(time_plan(plan, (M.data_ptr(), X.data_ptr(), Y.data_ptr()), stream, 7))
        d = plan.describe()
        print(f"{R}x{C} K={K} {v} {p} U={d['unroll']} xs={d['xmode']} smem={d['smem']} cps={d['ctas_per_sm']} "
              f"grid={d['grid']} {nbytes / us / 1e3:.0f} GB/s", flush=True)
    adaptic.clear_cache()
    del M
