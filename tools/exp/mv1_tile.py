"""Single-vector MV: x-tile stream-K kernel (XSMEM 3) vs the selector's pick (JSON lines)."""
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
X = torch.empty(1 << 24, device=dev); synth.device_vector(X, "uniform", 4)
Y = torch.empty(1 << 24, device=dev)
for k in range(3, 19):
    R, C = 1 << k, 1 << (26 - k)
    cands = [("AUTO", None)]
    for cw in (0, 2048, 4096, 8192, 16384):
        if cw <= C:
            for mb in (0, 16):
                for cps in (0, 1):
                    cands.append(("MV_SPLIT", [cw, 0, cps, 0, 3, 0, mb]))
    for v, p in cands:
        try:
            plan = adaptic.get_plan(L.OP_MV, R, C, L.F32, dev, v, p, stream)
        except adaptic.AdapticError:
            continue
        ts = time_plan(plan, (M.data_ptr(), X.data_ptr(), Y.data_ptr()), stream, 9)
        med = statistics.median(ts)
        d = plan.describe()
        print(json.dumps({"R": R, "C": C, "req": v, "params": p, "variant": d["variant"], "xmode": d["xmode"],
                          "us": med, "GBps": 4 * (R * C + R + C) / med / 1e3}), flush=True)
    adaptic.clear_cache()
