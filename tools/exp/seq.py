"""Does a kernel's time depend on what ran before it?  Time problem B after A (events around B)."""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_pldi_samadihmlm12_b200 as adaptic  # noqa: E402
from paper_conf_pldi_samadihmlm12_b200 import _lib as L  # noqa: E402

dev = torch.device("cuda:0")
stream = torch.cuda.current_stream().cuda_stream


def prob(op, R, C, variant="AUTO", params=None):
    M = torch.empty(R * C, device=dev)
    synth.device_matrix(M, R, C, "tmv" if op == "tmv" else "mv", "uniform", 1)
    X = torch.empty(C, device=dev)
    synth.device_vector(X, "uniform", 2)
    y = torch.empty(R, device=dev)
    plan = adaptic.get_plan({"mv": L.OP_MV, "tmv": L.OP_TMV}[op], R, C, L.F32, dev, variant, params, stream)
    return plan, (M.data_ptr(), X.data_ptr(), y.data_ptr()), (M, X, y)


def timeB(A, B, reps=20):
    ts = []
    for _ in range(reps):
        if A is not None:
            A[0].run(*A[1], stream)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        B[0].run(*B[1], stream)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    return statistics.median(ts)


tmv16 = prob("tmv", 1 << 22, 16)
mv8 = prob("mv", 1 << 23, 8)
mv8b = prob("mv", 1 << 23, 8, "MV_SUBWARP", [2, 0, 0, 1])
mv8c = prob("mv", 1 << 23, 8, "MV_SUBWARP", [1, 0, 0, 1, 1])
cpr = prob("mv", 1024, 65536)
tmv1024 = prob("tmv", 512, 131072)
mv2048 = prob("mv", 2048, 32768)
print("mv8 plan", mv8[0].describe())
for name, A, B in [("mv8 alone", None, mv8), ("tmv16 -> mv8", tmv16, mv8), ("mv8 -> mv8", mv8, mv8),
                   ("mv8b(G2) alone", None, mv8b), ("tmv16 -> mv8b", tmv16, mv8b),
                   ("mv8c(G1,ldg) alone", None, mv8c), ("tmv16 -> mv8c", tmv16, mv8c),
                   ("cpr alone", None, cpr), ("tmv512 -> cpr", tmv1024, cpr), ("mv2048 -> cpr", mv2048, cpr),
                   ("cpr -> cpr", cpr, cpr)]:
    print(f"{name:22s} {timeB(A, B):7.1f} us")

import time  # noqa: E402
for name, P in [("cpr", cpr), ("mv8", mv8), ("tmv16", tmv16)]:
    torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(200):
        P[0].run(*P[1], stream)
    host = (time.perf_counter() - t) / 200 * 1e6
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(20):
        P[0].run(*P[1], stream)
    e1.record()
    torch.cuda.synchronize()
    print(f"{name}: host {host:.1f} us/launch, b2b GPU {e0.elapsed_time(e1) * 1e3 / 20:.1f} us/launch")
