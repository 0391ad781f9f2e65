"""Why does the same CPR plan run at 51 us in the sweep and 76 us in seq.py?  Controlled A/B."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_pldi_samadihmlm12_b200 as adaptic  # noqa: E402
from paper_conf_pldi_samadihmlm12_b200 import _lib as L  # noqa: E402

dev = torch.device("cuda:0")
stream = torch.cuda.current_stream().cuda_stream
R, C = 1024, 65536
plan = adaptic.get_plan(L.OP_MV, R, C, L.F32, dev, "MV_CPR", [256, 0, 0, 2, 0, 0, 2], stream)
plan2 = adaptic.get_plan(L.OP_MV, R, C, L.F32, dev, "MV_CPR", [256, 0, 0, 4, 0, 0, 1], stream)


def b2b(p, ptrs, n=20):
    for _ in range(3):
        p.run(*ptrs, stream)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(n):
        p.run(*ptrs, stream)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3 / n


def show(tag, M, X, Y):
    for name, p in (("rb2u2", plan), ("rb1u4", plan2)):
        print(f"{tag:40s} {name}: {b2b(p, (M.data_ptr(), X.data_ptr(), Y.data_ptr())):6.1f} us")


M = torch.empty(R * C, device=dev)
X = torch.empty(C, device=dev)
Y = torch.empty(R, device=dev)
synth.device_matrix(M, R, C, "mv", "uniform", 1)
synth.device_vector(X, "uniform", 2)
show("own buffers, first allocation", M, X, Y)
Mz = torch.zeros(R * C, device=dev)
show("zero-filled A", Mz, X, Y)
Mo = torch.ones(R * C, device=dev)
show("all-ones A", Mo, X, Y)
big = [torch.empty(1 << 26, device=dev) for _ in range(12)]
show("own buffers after 3 GiB more allocated", M, X, Y)
Xbig = torch.empty(8 << 20, device=dev)
synth.device_vector(Xbig, "uniform", 2)
show("x = slice of a 32 MB buffer", M, Xbig, Y)
M2 = torch.empty(R * C, device=dev)
synth.device_matrix(M2, 1, R * C, "mv", "uniform", 11)
show("A filled like the sweep (seed 11, 1 x RC)", M2, X, Y)
Mr = torch.randn(R * C, device=dev)
show("A = randn", Mr, X, Y)
