"""Compare multi-vector MV kernels on 256 MiB shapes (experiment; JSON lines to stdout)."""
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
X = torch.empty(8 << 21, device=dev); synth.device_vector(X, "uniform", 4)
Y = torch.empty(8 << 23, device=dev)
shapes = [(1 << k, 1 << (26 - k)) for k in (3, 6, 8, 10, 12, 13, 14, 16, 18)]
for K in (2, 4, 8):
    for R, C in shapes:
        cands = [("AUTO", None), ("MV_WPR", None), ("MV_CPR", [0, 0, 0, 2, 1]), ("MV_CPR", [0, 0, 0, 2, 2]),
                 ("MV_SPLIT", [0, 0, 0, 2, 1]), ("MV_SPLIT", [0, 0, 0, 0, 3])]
        for cw in (512, 1024, 2048, 4096, 8192):
            if K * cw * 4 <= 200 * 1024 and cw <= C:
                cands.append(("MV_SPLIT", [cw, 0, 0, 0, 3]))
        cands.append(("MV_SPLIT", [0, 0, 1, 0, 3]))
        for v, p in cands:
            try:
                plan = adaptic.get_plan(L.OP_MV, R, C, L.F32, dev, v, p, stream, K)
            except adaptic.AdapticError as e:
                continue
            ts = time_plan(plan, (M.data_ptr(), X.data_ptr(), Y.data_ptr()), stream, 7)
            med = statistics.median(ts)
            b = 4 * (R * C + K * (R + C))
            d = plan.describe()
            print(json.dumps({"K": K, "R": R, "C": C, "req": v, "params": p, "variant": d["variant"], "xmode": d.get("xmode"),
                              "us": med, "GBps": b / med / 1e3, "grid": d.get("grid"), "lanes": d.get("lanes"), "rb": d.get("rb")}), flush=True)
        adaptic.clear_cache()
