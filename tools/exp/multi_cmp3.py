"""TMV multi-vector: TMA-staged vs register-fed kernels (JSON lines)."""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch
import synth
import paper_conf_pldi_samadihmlm12_b200 as adaptic
from paper_conf_pldi_samadihmlm12_b200 import _lib as L
from tools.sweep import time_plan
dev = torch.device("cuda:0")
stream = torch.cuda.current_stream().cuda_stream
N = 1 << 26
M = torch.empty(N, device=dev); synth.device_matrix(M, 1, N, "mv", "uniform", 3)
X = torch.empty(8 << 23, device=dev); synth.device_vector(X, "uniform", 4)
Y = torch.empty(8 << 23, device=dev)
shapes = [(1 << k, 1 << (26 - k)) for k in (6, 8, 10, 12, 13, 14, 16, 18, 20)]
for K in (4, 2, 8):
    for R, C in shapes:
        cands = [("AUTO", None), ("TMV_SPLITK", [0, 0, 0, 0, 1]), ("TMV_COL", None), ("TMV_REGTILE", [0, 0, 0, 0, 1])]
        if os.environ.get("MULTI_AUTO_ONLY"):
            cands = [("AUTO", None)]
        for lr in (() if os.environ.get("MULTI_AUTO_ONLY") else (16, 32, 64, 128, 256)):
            if lr * 4 <= max(64, R):
                for sp in (0, 9, 18, 37, 74, 148, 296):
                    cands.append(("TMV_SPLITK", [lr, sp, 0, 0, 0]))
        for v, p in cands:
            try:
                plan = adaptic.get_plan(L.OP_TMV, R, C, L.F32, dev, v, p, stream, K)
            except adaptic.AdapticError:
                continue
            ts = time_plan(plan, (M.data_ptr(), X.data_ptr(), Y.data_ptr()), stream, 7)
            med = statistics.median(ts)
            d = plan.describe()
            b = 4 * (R * C + K * (R + C))
            print(json.dumps({"K": K, "R": R, "C": C, "req": v, "params": p, "variant": d["variant"], "xmode": d["xmode"],
                              "lanes": d["lanes"], "splits": d["splits"], "grid": d["grid"], "us": med, "GBps": b / med / 1e3}), flush=True)
        adaptic.clear_cache()
