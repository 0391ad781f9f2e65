"""TMV with rows off the 16-byte grid on the constant-shift kernel (tmv_mis_kernel.cuh
tmv_shift_kernel; TMV_SPLITK with param XSMEM = 7) against the oracle -- needs a GPU.

R % 4 != 0 at every B base alignment (the word shift of a c-lane's rows is constant only
because the c-lane count is a multiple of 4: a wrong shift bookkeeping fails every case),
tiles of 4 LR - 4 outputs with a ragged last tile, splits (ticket merge), int32 (exact) and
integer-valued fp32 (P5, exact).  fp32: |y - y_ref| <= 1e-4 S_r per output."""
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
SHAPES = [(9, 1000), (61, 7), (63, 5003), (65, 100000), (251, 1), (253, 4097), (509, 3001), (1025, 2000),
          (2049, 513), (8193, 65), (30001, 33), (9, 77777)]
PARAMS = [[0, 0, 0, 0, 7], [16, 0, 0, 2, 7], [32, 3, 0, 4, 7], [64, 0, 0, 8, 7], [64, 17, 0, 2, 7]]


def placed(a, off, dtype):
    buf = torch.zeros(a.size + 8, dtype=dtype, device=DEV)
    buf[off:off + a.size] = torch.from_numpy(a.reshape(-1)).to(DEV)
    return buf[off:off + a.size].view(a.shape)


def test_tshift_every_shape_alignment_and_params():
    fails = []
    for (R, C), off, p in itertools.product(SHAPES, (0, 1, 2, 3), PARAMS):
        B = synth.matrix(R, C, "tmv", np.float32, "uniform", 61 + R)
        x = synth.vector(C, np.float32, "uniform", 62 + C)
        try:
            d = adaptic.plan("tmv", R, C, variant="TMV_SPLITK", params=p).describe()
            assert d["xmode"] == 7, d
            y = adaptic.tmv(placed(B, off, torch.float32), placed(x, (off + 1) % 4, torch.float32),
                            variant="TMV_SPLITK", params=p).cpu().numpy()
            yr, S = oracle.tmv(B, x)
            bad = ~(np.abs(y.astype(np.float64) - yr) <= 1e-4 * S)
            assert not bad.any(), f"{bad.sum()} outputs out of tolerance, first {np.argwhere(bad)[:4].ravel()}"
        except Exception as e:  # noqa: BLE001 -- report every failing case at once
            fails.append(f"{R}x{C} off={off} {p}: {type(e).__name__}: {str(e)[:160]}")
    assert not fails, f"{len(fails)} failures\n" + "\n".join(fails[:30])


def test_tshift_int32_and_p5_exact():
    for (R, C), off in itertools.product(((9, 100000), (1025, 3000), (8193, 500)), (0, 3)):
        B = synth.matrix(R, C, "tmv", np.int32, "uniform", 7 + R)
        x = synth.vector(C, np.int32, "uniform", 8 + R)
        y = adaptic.tmv(placed(B, off, torch.int32), torch.from_numpy(x).to(DEV), variant="TMV_SPLITK",
                        params=[0, 0, 0, 0, 7]).cpu().numpy()
        assert np.array_equal(y, oracle.tmv(B, x)), (R, C, off)
        Bf = synth.matrix(R, C, "tmv", np.float32, "smallint", 9 + R)
        xf = synth.vector(C, np.float32, "smallint", 10 + R)
        yf = adaptic.tmv(placed(Bf, off, torch.float32), torch.from_numpy(xf).to(DEV), variant="TMV_SPLITK",
                         params=[32, 5, 0, 4, 7]).cpu().numpy()
        assert np.array_equal(yf.astype(np.float64), oracle.tmv(Bf, xf)[0]), (R, C, off)


def test_window_kernel_every_shape_alignment_and_split():
    """tmv_window_kernel (TMV_SPLITK with XSMEM 10): one aligned 128-bit load per row and
    thread, 7 accumulators with a compile-time shift pattern per 4 rows (every R mod 4 and B
    base alignment), the halo shuffle between windows and tiles, rows left over after the
    groups of 4 / 8, splits with the ticket merge; with one split (S = 1) the warp-tile form
    (31 windows per warp, halo by shuffle, 128-bit y stores when y is aligned) at 2 and 3
    resident CTAs; fp32 within 1e-4 S_r, int32 exact."""
    fails = []
    shapes = SHAPES + [(1021, 3), (1022, 13), (1023, 300), (250000, 9), (8193, 1)]
    for (R, C), off, p in itertools.product(shapes, (0, 1, 2, 3),
                                            [[0, 0, 0, 0, 10], [0, 0, 0, 4, 10], [0, 7, 0, 8, 10],
                                             [0, 1, 0, 4, 10], [0, 1, 0, 8, 10], [0, 1, 3, 4, 10]]):
        for dt in ("f32", "i32"):
            np_dt = np.float32 if dt == "f32" else np.int32
            tdt = torch.float32 if dt == "f32" else torch.int32
            B = synth.matrix(R, C, "tmv", np_dt, "uniform", 71 + R)
            x = synth.vector(C, np_dt, "uniform", 72 + C)
            try:
                d = adaptic.plan("tmv", R, C, dt, variant="TMV_SPLITK", params=p).describe()
                if R % 4 == 0 or R < 8:
                    continue
                assert d["xmode"] == 10, d
                assert (d["lanes"] == 31) == (d["splits"] == 1), d
                y = adaptic.tmv(placed(B, off, tdt), placed(x, (off + 2) % 4, tdt), variant="TMV_SPLITK",
                                params=p).cpu().numpy()
                if dt == "i32":
                    assert np.array_equal(y, oracle.tmv(B, x)), "int32 mismatch"
                else:
                    yr, S = oracle.tmv(B, x)
                    bad = ~(np.abs(y.astype(np.float64) - yr) <= 1e-4 * S)
                    assert not bad.any(), f"{bad.sum()} out of tolerance, first {np.argwhere(bad)[:4].ravel()}"
            except Exception as e:  # noqa: BLE001
                fails.append(f"{dt} {R}x{C} off={off} {p}: {type(e).__name__}: {str(e)[:160]}")
    assert not fails, f"{len(fails)} failures\n" + "\n".join(fails[:30])
