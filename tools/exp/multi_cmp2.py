"""Few-row multi-vector MV: row stride / chunk / ticket-rows experiments (JSON lines)."""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch
import synth
import paper_conf_pldi_samadihmlm12_b200 as adaptic
from paper_conf_pldi_samadihmlm12_b200 import _lib as L
from tools.sweep import time_plan
dev = torch.device("cuda:0")
stream = torch.cuda.current_stream().cuda_stream
N = (1 << 26) + (1 << 12)
M = torch.empty(N, device=dev); synth.device_matrix(M, 1, N, "mv", "uniform", 3)
X = torch.empty(8 << 21, device=dev); synth.device_vector(X, "uniform", 4)
Y = torch.empty(8 << 23, device=dev)
for K in (2, 4):
    for R, C in [(64, 1 << 20), (64, (1 << 20) + 4), (64, (1 << 20) + 64), (8, 1 << 23), (8, (1 << 23) + 4), (256, 1 << 18), (256, (1 << 18) + 4)]:
        cands = [("AUTO", None), ("MV_SPLIT", [0, 0, 0, 2, 1])]
        for cw in (1024, 2048, 4096):
            for mb in (0, 8, 64):
                cands.append(("MV_SPLIT", [cw, 0, 0, 0, 3, 0, mb]))
        cands.append(("MV_SPLIT", [2048, 0, 1, 0, 3, 0, 0]))
        for v, p in cands:
            try:
                plan = adaptic.get_plan(L.OP_MV, R, C, L.F32, dev, v, p, stream, K)
            except adaptic.AdapticError:
                continue
            ts = time_plan(plan, (M.data_ptr(), X.data_ptr(), Y.data_ptr()), stream, 7)
            med = statistics.median(ts)
            b = 4 * (R * C + K * (R + C))
            print(json.dumps({"K": K, "R": R, "C": C, "req": v, "params": p, "us": med, "GBps": b / med / 1e3}), flush=True)
        adaptic.clear_cache()
