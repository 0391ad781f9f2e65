"""TMV with B staged by TMA (tmv_ring_kernel.cuh; TMV variants with param XSMEM = 6), K = 1,
2, 4, 8 vectors, against the oracle -- needs a GPU.

Covers: one tile of whole rows (R <= tile width: one contiguous bulk copy per stage) and
many tiles of row segments, R off the 16-byte grid (rows at word shifts 1..3), base
pointers that are only 4-byte aligned (B's unaligned first / last words read from global
memory), a ragged last tile, c-lane sums, tiles spread over many CTAs (ticket merge),
stage counts, int32 (K = 1, bit-exact) and integer-valued fp32 (P5, bit-exact and
deterministic).  fp32: |y - y_ref| <= 1e-4 S_r per output."""
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
SHAPES = [(1, 1), (3, 5), (64, 1000), (65, 7777), (129, 40000), (1000, 33), (1025, 3000), (2048, 100),
          (4100, 77), (8192, 64), (9000, 13), (3, 300000), (33000, 9)]
RING = [0, 0, 0, 0, 6]


def check(Y, B, X, what):
    for j in range(X.shape[0]):
        yr, S = oracle.tmv(B, X[j])
        bad = ~(np.abs(Y[j].astype(np.float64) - yr) <= 1e-4 * S)
        assert not bad.any(), f"{what} vector {j}: {bad.sum()} outputs out of tolerance"


def run(Bd, Xd, K, params=RING):
    if K == 1:
        return adaptic.tmv(Bd, Xd[0], variant="TMV_SPLITK", params=params).cpu().numpy()[None, :]
    return adaptic.tmv_multi(Bd, Xd, variant="TMV_SPLITK", params=params).cpu().numpy()


@pytest.mark.parametrize("K", [1, 2, 4, 8])
def test_tring_every_shape_and_alignment(K):
    fails = []
    for (R, C), off in itertools.product(SHAPES, (0, 1, 3)):
        B = synth.matrix(R, C, "tmv", np.float32, "uniform", 91 + R)
        X = synth.matrix(K, C, "mv", np.float32, "uniform", 92 + C)
        Bb = torch.zeros(B.size + 8, device=DEV)
        Bb[off:off + B.size] = torch.from_numpy(B.reshape(-1)).to(DEV)
        Xb = torch.zeros(X.size + 8, device=DEV)
        Xb[off:off + X.size] = torch.from_numpy(X.reshape(-1)).to(DEV)
        Bd, Xd = Bb[off:off + B.size].view(C, R), Xb[off:off + X.size].view(K, C)
        for params in (RING, RING + [0, 0, 0, 2], [1] + RING[1:], [2] + RING[1:]):
            try:
                d = adaptic.plan("tmv", R, C, variant="TMV_SPLITK", params=params, nvec=K).describe()
                assert d["xmode"] == 6, d
                check(run(Bd, Xd, K, params), B, X, f"K={K} {R}x{C} off={off} {params}")
            except Exception as e:  # noqa: BLE001 -- report every failing case at once
                fails.append(f"K={K} {R}x{C} off={off} {params}: {type(e).__name__}: {str(e)[:200]}")
    assert not fails, f"{len(fails)} failures\n" + "\n".join(fails[:30])


def test_tring_int32_and_p5_exact():
    for R, C in ((257, 5000), (4097, 300), (1000, 65536), (7, 1 << 20)):
        B = synth.matrix(R, C, "tmv", np.int32, "uniform", 5 + R)
        x = synth.vector(C, np.int32, "uniform", 6 + R)
        y = adaptic.tmv(torch.from_numpy(B).to(DEV), torch.from_numpy(x).to(DEV), variant="TMV_SPLITK",
                        params=RING).cpu().numpy()
        assert np.array_equal(y, oracle.tmv(B, x)), (R, C)
    R, C = 1025, 50000
    B = synth.matrix(R, C, "tmv", np.float32, "smallint", 7)
    X = synth.matrix(4, C, "mv", np.float32, "smallint", 8)
    Bd, Xd = torch.from_numpy(B).to(DEV), torch.from_numpy(X).to(DEV)
    Y1, Y2 = run(Bd, Xd, 4), run(Bd, Xd, 4)
    assert np.array_equal(Y1, Y2)
    for j in range(4):
        assert np.array_equal(Y1[j].astype(np.float64), oracle.tmv(B, X[j])[0])
