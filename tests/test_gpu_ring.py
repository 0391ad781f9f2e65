"""MV with the matrix staged by TMA (mmv_ring_kernel.cuh; MV_CPR / MV_SPLIT with param
XSMEM = 6), K = 1, 2, 4, 8 vectors, against the oracle -- needs a GPU.

Covers: groups of 8 rows with a ragged last group, rows shorter than one 256-float4 stage,
x resident in shared memory (K C 4 <= 64 KB) and streamed with the stages, groups spread
over many CTAs (ticket merge) and many groups per CTA, the stage count (param PIPE), int32
(K = 1, bit-exact), integer-valued fp32 data (P5: bit-exact, deterministic), and 4-byte-
aligned pointers (the planned fallbacks).  fp32: |y - y_ref| <= 1e-4 S_r per output."""
import itertools

import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_pldi_samadihmlm12_b200 as adaptic

DEV = "cuda:0"
SHAPES = [(1, 4), (3, 1024), (8, 40000), (9, 4100), (17, 2048), (64, 65536), (100, 1028), (1000, 2048),
          (4100, 256), (2, 1 << 20), (333, 16388)]
RING = [0, 0, 0, 0, 6]


def check(Y, A, X, what):
    for j in range(X.shape[0]):
        yr, S = oracle.mv(A, X[j])
        bad = ~(np.abs(Y[j].astype(np.float64) - yr) <= 1e-4 * S)
        assert not bad.any(), f"{what} vector {j}: {bad.sum()} rows out of tolerance"


def run(A, X, variant="MV_SPLIT", params=RING):
    Ad, Xd = torch.from_numpy(A).to(DEV), torch.from_numpy(X).to(DEV)
    if X.shape[0] == 1:
        return adaptic.mv(Ad, Xd[0], variant=variant, params=params).cpu().numpy()[None, :]
    return adaptic.mv_multi(Ad, Xd, variant=variant, params=params).cpu().numpy()


@pytest.mark.parametrize("K", [1, 2, 4, 8])
def test_ring_every_shape(K):
    fails = []
    for (R, C), (v, p) in itertools.product(SHAPES, [("MV_SPLIT", RING), ("MV_CPR", RING + [0, 0, 0, 2])]):
        A = synth.matrix(R, C, "mv", np.float32, "uniform", 81 + R)
        X = synth.matrix(K, C, "mv", np.float32, "uniform", 82 + C)
        try:
            d = (adaptic.plan("mv", R, C, variant=v, params=p, nvec=K)).describe()
            assert d["xmode"] == 6, d
            check(run(A, X, v, p), A, X, f"K={K} {R}x{C} {v} {p}")
        except Exception as e:  # noqa: BLE001 -- report every failing case at once
            fails.append(f"K={K} {R}x{C} {v}: {type(e).__name__}: {str(e)[:200]}")
    assert not fails, "\n".join(fails)


def test_ring_int32_and_p5_exact_and_deterministic():
    for R, C in ((40, 4096), (300, 50000), (7, 1 << 20), (2049, 1028)):
        A = synth.matrix(R, C, "mv", np.int32, "uniform", 11 + R)
        x = synth.vector(C, np.int32, "uniform", 12 + R)
        y = adaptic.mv(torch.from_numpy(A).to(DEV), torch.from_numpy(x).to(DEV), variant="MV_SPLIT",
                       params=RING).cpu().numpy()
        assert np.array_equal(y, oracle.mv(A, x)), (R, C)
    R, C = 300, 50000
    A = synth.matrix(R, C, "mv", np.float32, "smallint", 5)
    X = synth.matrix(4, C, "mv", np.float32, "smallint", 6)
    Y1, Y2 = run(A, X), run(A, X)
    assert np.array_equal(Y1, Y2)
    for j in range(4):
        assert np.array_equal(Y1[j].astype(np.float64), oracle.mv(A, X[j])[0])


@pytest.mark.parametrize("K", [1, 4])
def test_ring_4byte_aligned_pointers_fall_back(K):
    R, C = 64, 8192
    A = synth.matrix(R, C, "mv", np.float32, "uniform", 9)
    X = synth.matrix(K, C, "mv", np.float32, "uniform", 10)
    big = torch.zeros(R * C + 4, device=DEV)
    big[1:1 + R * C] = torch.from_numpy(A.reshape(-1)).to(DEV)
    xb = torch.zeros(K * C + 4, device=DEV)
    xb[1:1 + K * C] = torch.from_numpy(X.reshape(-1)).to(DEV)
    Am, Xm = big[1:1 + R * C].view(R, C), xb[1:1 + K * C].view(K, C)
    if K == 1:
        Y = adaptic.mv(Am, Xm[0], variant="MV_SPLIT", params=RING).cpu().numpy()[None, :]
    else:
        Y = adaptic.mv_multi(Am, Xm, variant="MV_SPLIT", params=RING).cpu().numpy()
    check(Y, A, X, "4-byte aligned")


def test_ring_reruns_identical_and_workspace_rearmed():
    """Tickets re-arm: repeated runs of the same plan (groups over many CTAs) are identical."""
    R, C = 16, 1 << 20
    A = synth.matrix(R, C, "mv", np.float32, "uniform", 3)
    X = synth.matrix(8, C, "mv", np.float32, "uniform", 4)
    Ad, Xd = torch.from_numpy(A).to(DEV), torch.from_numpy(X).to(DEV)
    ys = [adaptic.mv_multi(Ad, Xd, variant="MV_SPLIT", params=RING).cpu().numpy() for _ in range(3)]
    assert np.array_equal(ys[0], ys[1]) and np.array_equal(ys[1], ys[2])
    check(ys[0], A, X, "rerun")
