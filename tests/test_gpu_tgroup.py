"""TMV with rows off the 16-byte grid on groups of four rows (tmv_group_kernel.cuh; TMV_REGTILE /
TMV_SPLITK with param XSMEM = 12) against the oracle -- needs a GPU.

Four rows of B are R whole 128-bit vectors, so thread slot v keeps the outputs (4v + j) mod R and
the row offsets (4v + j) div R for the whole kernel: a wrong offset, a wrong x row at the row
boundary inside a vector, a dropped sub-group, a lost tail row (C mod 4) or a broken two-level
merge fails one of these.  Every R mod 4, sub-groups per CTA step (R < threads) and several
slots per thread (R > 1024, or forced), contiguous and interleaved CTA group order, C with
every remainder mod 4, grids from one CTA to many (more
than one 16-CTA merge group), B at every 4-byte offset (offsets 1..3 run the TMV_SPLITK
fallback), fp32 within 1e-4 S_r, int32 exact, integer-valued fp32 (P5) exact."""
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
SHAPES = [(5, 4003), (9, 1000), (17, 100001), (33, 7), (63, 5002), (65, 300003), (129, 1), (255, 40001),
          (257, 3), (513, 20002), (1023, 999), (1025, 40003), (1537, 2), (2049, 9001), (2559, 1234)]
PARAMS = [[0, 0, 0, 0, 12], [0, 0, 0, 8, 12], [0, 0, 1, 0, 12], [0, 0, 0, 0, 12, 512],
          [0, 0, 0, 0, 12, 0, 0, 2], [0, 0, 0, 0, 12, 0, 2, 2], [0, 0, 0, 2, 12, 0, 4, 1]]


def placed(a, off, dtype):
    buf = torch.zeros(a.size + 8, dtype=dtype, device=DEV)
    buf[off:off + a.size] = torch.from_numpy(a.reshape(-1)).to(DEV)
    return buf[off:off + a.size].view(a.shape)


def _params(p):
    return (p + [0] * 9)[:9]


def test_group_kernel_every_shape_alignment_and_params():
    fails = []
    for (R, C), off, p in itertools.product(SHAPES, (0, 1, 3), PARAMS):
        for variant in ("TMV_REGTILE", "TMV_SPLITK"):
            pp = _params(p)
            try:
                pl = adaptic.plan("tmv", R, C, variant=variant, params=pp)
            except Exception:  # noqa: BLE001 -- a forced (U, block, slots) not valid for this R
                if pp[3] or pp[5] or pp[6]:
                    continue
                raise
            d = pl.describe()
            assert d["xmode"] == 12, d
            B = synth.matrix(R, C, "tmv", np.float32, "uniform", 81 + R)
            x = synth.vector(C, np.float32, "uniform", 82 + C)
            try:
                y = adaptic.tmv(placed(B, off, torch.float32), placed(x, (off + 1) % 4, torch.float32),
                                variant=variant, params=pp).cpu().numpy()
                yr, S = oracle.tmv(B, x)
                bad = ~(np.abs(y.astype(np.float64) - yr) <= 1e-4 * S)
                assert not bad.any(), f"{bad.sum()} outputs out of tolerance, first {np.argwhere(bad)[:4].ravel()}"
            except Exception as e:  # noqa: BLE001 -- report every failing case at once
                fails.append(f"{variant} {R}x{C} off={off} {pp}: {type(e).__name__}: {str(e)[:160]}")
    assert not fails, f"{len(fails)} failures\n" + "\n".join(fails[:30])


def test_group_kernel_int32_and_p5_exact():
    for (R, C) in ((9, 100003), (257, 5001), (1025, 3002), (2049, 777)):
        B = synth.matrix(R, C, "tmv", np.int32, "uniform", 7 + R)
        x = synth.vector(C, np.int32, "uniform", 8 + R)
        y = adaptic.tmv(torch.from_numpy(B).to(DEV), torch.from_numpy(x).to(DEV), variant="TMV_SPLITK",
                        params=_params([0, 0, 0, 0, 12])).cpu().numpy()
        assert np.array_equal(y, oracle.tmv(B, x)), (R, C)
        Bf = synth.matrix(R, C, "tmv", np.float32, "smallint", 9 + R)
        xf = synth.vector(C, np.float32, "smallint", 10 + R)
        yf = adaptic.tmv(torch.from_numpy(Bf).to(DEV), torch.from_numpy(xf).to(DEV), variant="TMV_REGTILE",
                         params=_params([0, 0, 0, 0, 12])).cpu().numpy()
        assert np.array_equal(yf.astype(np.float64), oracle.tmv(Bf, xf)[0]), (R, C)


def test_group_kernel_reruns_identical_and_bench_shapes():
    """Deterministic merge (same bits on a rerun, the workspace re-armed) and the offgrid bench's
    R + 1 shapes at full size on sampled outputs."""
    for R, C in ((17, 1 << 22), (513, 1 << 17), (1025, 1 << 16), (2049, 1 << 15)):
        B = torch.empty(C, R, dtype=torch.float32, device=DEV).uniform_(-1, 1)
        x = torch.empty(C, dtype=torch.float32, device=DEV).uniform_(-1, 1)
        p = _params([0, 0, 0, 0, 12])
        y1 = adaptic.tmv(B, x, variant="TMV_SPLITK", params=p)
        y2 = adaptic.tmv(B, x, variant="TMV_SPLITK", params=p)
        assert torch.equal(y1, y2), (R, C)
        Bh, xh = B.cpu().numpy(), x.cpu().numpy()
        yh = y1.cpu().numpy()
        for r in (0, 1, R // 2, R - 2, R - 1):
            col = Bh[:, r].astype(np.float64)
            ref = float(np.dot(col, xh.astype(np.float64)))
            S = float(np.dot(np.abs(col), np.abs(xh.astype(np.float64))))
            assert abs(float(yh[r]) - ref) <= 1e-4 * S, (R, C, r)
