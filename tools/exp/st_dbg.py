import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import synth, oracle
import paper_conf_pldi_samadihmlm12_b200 as adaptic
for (H, W) in [(1, 4), (2, 8), (64, 256)]:
    for p in ([0, 0, 0, 0, 0, 0, 0, 2], [0, 0, 0, 0, 0, 0, 0, 3], None):
        u = synth.matrix(H, W, "mv", np.float32, "uniform", 41 + H + W)
        out = adaptic.stencil5(torch.from_numpy(u).to("cuda:0"), 0.6, 0.1, variant="ST_DIRECT", params=p)
        torch.cuda.synchronize()
        print(H, W, p, "ok", flush=True)
