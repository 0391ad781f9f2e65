"""MV with rows too long for x in registers on staged column chunks (rowtile_kernel.cuh
mv_chunk_cta_kernel; MV_CPR / MV_SPLIT with param XSMEM = 13) against the oracle -- needs a GPU.

Chunk j of row r starts (r C + j W) mod 4 words into its stage slot, so every C mod 4, chunk
widths that do not divide C, CTA unit ranges that cross chunk boundaries (x reloaded), 1-4 row
segments per tile with a ragged last tile, the matrix's last < 4 words copied by the threads,
one chunk (no merge) and hundreds of chunks (L-lane merge), A at every 4-byte offset (offsets
1..3 run the direct fallback); fp32 within 1e-4 S_r, int32 exact, integer-valued fp32 (P5)
exact, reruns bit-identical."""
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
SHAPES = [(1, 9), (3, 5000), (7, 100003), (13, 40001), (64, 33000), (129, 20002), (300, 9001), (1000, 4100),
          (2, 300007), (5, 8193)]
PARAMS = [[0, 0, 0, 0, 13], [8, 0, 0, 0, 13, 256], [8, 0, 0, 3, 13, 512, 4], [36, 0, 0, 0, 13],
          [16, 0, 2, 0, 13, 256, 2], [8, 0, 1, 2, 13, 256, -20]]


def placed(a, off, dtype):
    buf = torch.zeros(a.size + 8, dtype=dtype, device=DEV)
    buf[off:off + a.size] = torch.from_numpy(a.reshape(-1)).to(DEV)
    return buf[off:off + a.size].view(a.shape)


def _p(p):
    return (p + [0] * 9)[:9]


def test_chunk_kernel_every_shape_alignment_and_params():
    fails = []
    for (R, C), off, p in itertools.product(SHAPES, (0, 2), PARAMS):
        variant = "MV_SPLIT" if (R + C) % 2 else "MV_CPR"
        pp = _p(p)
        try:
            d = adaptic.plan("mv", R, C, variant=variant, params=pp).describe()
        except Exception:  # noqa: BLE001 -- a forced combination the ring budget cannot hold
            if pp[2] >= 2:
                continue
            raise
        assert d["xmode"] == 13, d
        A = synth.matrix(R, C, "mv", np.float32, "uniform", 91 + R)
        x = synth.vector(C, np.float32, "uniform", 92 + C)
        try:
            y = adaptic.mv(placed(A, off, torch.float32), placed(x, (off + 3) % 4, torch.float32),
                           variant=variant, params=pp).cpu().numpy()
            yr, S = oracle.mv(A, x)
            bad = ~(np.abs(y.astype(np.float64) - yr) <= 1e-4 * S)
            assert not bad.any(), f"{bad.sum()} rows out of tolerance, first {np.argwhere(bad)[:4].ravel()}"
        except Exception as e:  # noqa: BLE001 -- report every failing case at once
            fails.append(f"{variant} {R}x{C} off={off} {pp} nch={d['splits']} k={d['rows_per_group']}: "
                         f"{type(e).__name__}: {str(e)[:160]}")
    assert not fails, f"{len(fails)} failures\n" + "\n".join(fails[:30])


def test_chunk_kernel_int32_and_p5_exact():
    for (R, C) in ((9, 100001), (130, 20003), (2, 700001)):
        A = synth.matrix(R, C, "mv", np.int32, "uniform", 17 + R)
        x = synth.vector(C, np.int32, "uniform", 18 + R)
        y = adaptic.mv(torch.from_numpy(A).to(DEV), torch.from_numpy(x).to(DEV), variant="MV_SPLIT",
                       params=_p([8, 0, 0, 0, 13, 256])).cpu().numpy()
        assert np.array_equal(y, oracle.mv(A, x)), (R, C)
        Af = synth.matrix(R, C, "mv", np.float32, "smallint", 19 + R)
        xf = synth.vector(C, np.float32, "smallint", 20 + R)
        yf = adaptic.mv(torch.from_numpy(Af).to(DEV), torch.from_numpy(xf).to(DEV), variant="MV_CPR",
                        params=_p([0, 0, 0, 0, 13])).cpu().numpy()
        assert np.array_equal(yf.astype(np.float64), oracle.mv(Af, xf)[0]), (R, C)


def test_chunk_kernel_reruns_identical_and_bench_shapes():
    """The offgrid bench's long C + 1 rows at full size: bit-identical reruns (the ticket
    counter re-armed) and sampled rows against an fp64 dot product."""
    for R, C in ((16, (1 << 22) + 1), (512, (1 << 17) + 1), (2048, (1 << 15) + 1)):
        A = torch.empty(R, C, dtype=torch.float32, device=DEV).uniform_(-1, 1)
        x = torch.empty(C, dtype=torch.float32, device=DEV).uniform_(-1, 1)
        p = _p([0, 0, 0, 0, 13])
        y1 = adaptic.mv(A, x, variant="MV_SPLIT", params=p)
        y2 = adaptic.mv(A, x, variant="MV_SPLIT", params=p)
        assert torch.equal(y1, y2), (R, C)
        xh = x.cpu().numpy().astype(np.float64)
        yh = y1.cpu().numpy()
        for r in (0, 1, R // 2, R - 1):
            row = A[r].cpu().numpy().astype(np.float64)
            ref = float(np.dot(row, xh))
            S = float(np.dot(np.abs(row), np.abs(xh)))
            assert abs(float(yh[r]) - ref) <= 1e-4 * S, (R, C, r)
