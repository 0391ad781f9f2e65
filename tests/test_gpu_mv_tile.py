"""Single-vector fp32 MV on the x-tile stream-K kernel (mmv_tile_kernel with K = 1; param
XSMEM = 3) against the oracle -- needs a GPU.  Covers one and many column chunks, odd
merge-block sizes, ragged rows, pieces smaller than a warp's rows, and the fallback to the
CTA-per-row kernel when the pointers are only 4-byte aligned.  |y - y_ref| <= 1e-4 S_r."""
import itertools

import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_pldi_samadihmlm12_b200 as adaptic
    from paper_conf_pldi_samadihmlm12_b200 import _lib as L

DEV = "cuda:0"


def check(y, A, x, what):
    yr, S = oracle.mv(A, x)
    bad = ~(np.abs(y.astype(np.float64) - yr) <= 1e-4 * S)
    assert not bad.any(), f"{what}: {bad.sum()} rows out of tolerance, first {np.argwhere(bad)[:3].ravel().tolist()}"


SHAPES = [(1, 4), (3, 8), (5, 512), (33, 1024), (100, 4100), (7, 40000), (517, 1028), (64, 65536), (1000, 12)]
PARAMS = [[0, 0, 0, 0, 3], [128, 0, 0, 0, 3, 0, 1], [512, 0, 1, 0, 3, 0, 3], [4096, 0, 0, 0, 3, 0, 64],
          [16384, 0, 0, 0, 3, 0, 0]]


def test_tile_kernel_every_shape():
    fails = []
    for (R, C), p in itertools.product(SHAPES, PARAMS):
        A = synth.matrix(R, C, "mv", np.float32, "uniform", 71 + R)
        x = synth.vector(C, np.float32, "uniform", 72 + C)
        try:
            y = adaptic.mv(torch.from_numpy(A).to(DEV), torch.from_numpy(x).to(DEV), variant="MV_SPLIT", params=p)
            if C % 4 == 0:
                assert adaptic.plan("mv", R, C, variant="MV_SPLIT", params=p).describe()["xmode"] == 4
            check(y.cpu().numpy(), A, x, f"{R}x{C} {p}")
        except Exception as e:  # noqa: BLE001 -- report every failing case at once
            fails.append(f"{R}x{C} {p}: {type(e).__name__}: {str(e)[:160]}")
    assert not fails, "\n".join(fails)


def test_integer_data_exact_and_deterministic():
    R, C = 300, 50000
    A = synth.matrix(R, C, "mv", np.float32, "smallint", 5)
    x = synth.vector(C, np.float32, "smallint", 6)
    yr, _ = oracle.mv(A, x)
    Ad, xd = torch.from_numpy(A).to(DEV), torch.from_numpy(x).to(DEV)
    y1 = adaptic.mv(Ad, xd, variant="MV_SPLIT", params=[1024, 0, 0, 0, 3, 0, 2]).cpu().numpy()
    y2 = adaptic.mv(Ad, xd, variant="MV_SPLIT", params=[1024, 0, 0, 0, 3, 0, 2]).cpu().numpy()
    assert np.array_equal(y1.astype(np.float64), yr)
    assert np.array_equal(y1, y2)


def test_misaligned_pointers_fall_back():
    R, C = 64, 8192
    A = synth.matrix(R, C, "mv", np.float32, "uniform", 9)
    x = synth.vector(C, np.float32, "uniform", 10)
    big = torch.zeros(R * C + 4, device=DEV)
    big[1:1 + R * C] = torch.from_numpy(A.reshape(-1)).to(DEV)
    xb = torch.zeros(C + 4, device=DEV)
    xb[1:1 + C] = torch.from_numpy(x).to(DEV)
    y = adaptic.mv(big[1:1 + R * C].view(R, C), xb[1:1 + C], variant="MV_SPLIT", params=[0, 0, 0, 0, 3])
    check(y.cpu().numpy(), A, x, "misaligned")


def test_int32_tile_kernel_is_exact():
    """int32 (modulo 2^32) runs the same kernel; every order is exact, so bit-exact."""
    for R, C, p in ((40, 4096, [0, 0, 0, 0, 3]), (300, 50000, [256, 0, 0, 0, 3, 0, 3]), (7, 1 << 20, [0, 0, 0, 0, 3])):
        A = synth.matrix(R, C, "mv", np.int32, "uniform", 11 + R)
        x = synth.vector(C, np.int32, "uniform", 12 + R)
        assert adaptic.plan("mv", R, C, "i32", variant="MV_SPLIT", params=p).describe()["xmode"] == 4
        y = adaptic.mv(torch.from_numpy(A).to(DEV), torch.from_numpy(x).to(DEV), variant="MV_SPLIT",
                       params=p).cpu().numpy()
        assert np.array_equal(y, oracle.mv(A, x)), (R, C, p)
