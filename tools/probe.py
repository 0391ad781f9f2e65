#!/usr/bin/env python
"""Bandwidth ceilings on this box: torch copy / sum over 256 MiB-1 GiB, back-to-back,
CUDA events.  Context for the roofline (not a bench number)."""
import json
import statistics

import torch


def timeit(fn, reps=30):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) / 1e3)
    return statistics.median(ts)


for mib in (256, 1024, 4096):
    n = mib * (1 << 20) // 4
    A = torch.randn(n, device="cuda")
    B = torch.empty_like(A)
    t_copy = timeit(lambda: B.copy_(A))
    t_sum = timeit(lambda: A.sum())
    print(json.dumps({"MiB": mib, "copy_GBps": 2 * 4 * n / t_copy / 1e9, "sum_read_GBps": 4 * n / t_sum / 1e9}))
