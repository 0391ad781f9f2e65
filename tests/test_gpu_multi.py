"""Multi-vector MV / TMV (adaptic_plan_multi; horizontal actor integration)
against the oracle, one vector at a time -- needs a GPU.  fp32 within 1e-4 * S_r."""
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
TOL = 1e-4
MV_FORCED = [("AUTO", None)] + [("MV_SUBWARP", [g, 0, 0, u]) for g in (1, 4, 16) for u in (1, 2, 4)] + \
            [("MV_WPR", [0, 0, 0, u]) for u in (1, 2)] + [("MV_CPR", [0, 0, 0, u]) for u in (1, 2)] + \
            [("MV_SPLIT", [0, s, 0, 2]) for s in (2, 7)] + \
            [("MV_SPLIT", [0, 0, 0, 0, 3]), ("MV_SPLIT", [128, 0, 0, 0, 3, 0, 1]), ("MV_SPLIT", [256, 0, 1, 0, 3, 0, 3]),
             ("MV_CPR", [1024, 0, 0, 0, 3, 0, 64])]   # x-tile stream-K kernel: default, many chunks, odd MB
TMV_FORCED = [("AUTO", None), ("TMV_COL", None)] + [("TMV_SPLITK", [lr, s]) for lr in (1, 8, 64) for s in (0, 3)] + \
             [("TMV_REGTILE", None), ("TMV_SPLITK", [64, 0, 0, 0, 1]), ("TMV_SPLITK", [16, 5, 0, 0, 3]),
              ("TMV_SPLITK", [256, 3, 1, 0, 3]), ("TMV_SPLITK", [0, 0, 0, 0, 3]),
              ("TMV_REGTILE", [0, 0, 0, 0, 3])]    # register-fed kernel; TMA-staged (XSMEM 3)


def check(Y, M, X, op, what):
    for j in range(X.shape[0]):
        yr, S = (oracle.mv(M, X[j]) if op == "mv" else oracle.tmv(M, X[j]))
        err = np.abs(Y[j].astype(np.float64) - yr)
        bad = ~(err <= TOL * S)
        assert not bad.any(), f"{what} vector {j}: {bad.sum()} out of tolerance"


def _collect(cases):
    fails = []
    for what, fn in cases:
        try:
            fn()
        except Exception as e:  # noqa: BLE001 -- report every failing case at once
            fails.append(f"{what}: {type(e).__name__}: {str(e)[:200]}")
    assert not fails, f"{len(fails)} failures:\n" + "\n".join(fails[:40])


@pytest.mark.parametrize("op", ["mv", "tmv"])
@pytest.mark.parametrize("K", [2, 4, 8])
def test_every_variant(op, K):
    shapes = [(1, 1), (3, 5), (33, 64), (100, 257), (517, 1024), (7, 40000), (1000, 12), (64, 100), (5000, 8),
              (256, 40000), (1024, 3001), (2048, 17)]
    forced = MV_FORCED if op == "mv" else TMV_FORCED

    def case(R, C, v, p):
        M = synth.matrix(R, C, op, np.float32, "uniform", synth.seed(13, "A") + R + C)
        X = synth.matrix(K, C, "mv", np.float32, "uniform", synth.seed(13, "x") + C)
        try:
            fn = adaptic.mv_multi if op == "mv" else adaptic.tmv_multi
            Y = fn(torch.from_numpy(M).to(DEV), torch.from_numpy(X).to(DEV), variant=v, params=p)
        except adaptic.AdapticError as e:
            ok = (L.ERR_UNSUPPORTED, L.ERR_MISALIGNED)
            if p and len(p) > 3 and K * p[3] > 16:         # K x U x-vectors in registers: at most 16
                ok += (L.ERR_INVALID_ARG,)
            assert e.status in ok, str(e)
            return
        check(Y.cpu().numpy(), M, X, op, f"{op} K={K} {R}x{C} {v} {p}")
    _collect([(f"{R}x{C} {v} {p}", lambda R=R, C=C, v=v, p=p: case(R, C, v, p))
              for (R, C), (v, p) in itertools.product(shapes, forced)])


@pytest.mark.parametrize("K", [1, 3, 5, 7, 11])
def test_any_vector_count_is_chunked(K):
    """K not in {1, 2, 4, 8}: the binding covers it with library calls of 8/4/2/1 vectors."""
    for op, (R, C) in (("mv", (300, 2000)), ("tmv", (2000, 300))):
        M = synth.matrix(R, C, op, np.float32, "uniform", 17 + K)
        X = synth.matrix(K, C, "mv", np.float32, "uniform", 18 + K)
        fn = adaptic.mv_multi if op == "mv" else adaptic.tmv_multi
        check(fn(torch.from_numpy(M).to(DEV), torch.from_numpy(X).to(DEV)).cpu().numpy(), M, X, op, f"{op} K={K}")


def test_exact_on_integer_data_and_equal_to_single_calls():
    """P5: integer-valued data is exact for every vector; so multi == K single calls bit for bit."""
    for op, (R, C) in (("mv", (1000, 4096)), ("tmv", (4096, 1000)), ("mv", (64, 1 << 18))):
        M = synth.matrix(R, C, op, np.float32, "smallint", 3)
        X = synth.matrix(8, C, "mv", np.float32, "smallint", 4)
        Md, Xd = torch.from_numpy(M).to(DEV), torch.from_numpy(X).to(DEV)
        fn, single = (adaptic.mv_multi, adaptic.mv) if op == "mv" else (adaptic.tmv_multi, adaptic.tmv)
        Y = fn(Md, Xd).cpu().numpy()
        for j in range(8):
            assert np.array_equal(Y[j], single(Md, Xd[j]).cpu().numpy()), (op, j)
            assert np.array_equal(Y[j].astype(np.float64), (oracle.mv(M, X[j]) if op == "mv" else oracle.tmv(M, X[j]))[0])


def test_device_generated_256MiB():
    for op, (R, C), K in (("mv", (4096, 16384), 4), ("tmv", (16384, 4096), 4), ("mv", (64, 1 << 20), 4),
                          ("mv", (64, 1 << 20), 8), ("mv", (8192, 8192), 2), ("mv", (65536, 1024), 8),
                          ("tmv", (64, 1 << 20), 4), ("tmv", (8192, 8192), 8), ("tmv", (1 << 20, 64), 2)):
        t = torch.empty(R * C, dtype=torch.float32, device=DEV)
        synth.device_matrix(t, R, C, op, "uniform", synth.seed(14, "A"))
        M = t.cpu().numpy().reshape((R, C) if op == "mv" else (C, R))
        X = synth.matrix(K, C, "mv", np.float32, "uniform", 15)
        fn = adaptic.mv_multi if op == "mv" else adaptic.tmv_multi
        Y = fn(t.view(M.shape), torch.from_numpy(X).to(DEV)).cpu().numpy()
        check(Y, M, X, op, f"{op} {R}x{C} K={K} 256MiB")


@pytest.mark.parametrize("op", ["mv", "tmv"])
@pytest.mark.parametrize("K", [2, 4, 8])
def test_4byte_aligned_pointers_fall_back(op, K):
    """only non-4-byte-aligned pointers are errors.  A 128-bit-shape multi plan
    (AUTO: x tiles / TMA tiles / register-x lane groups) run on 4-byte-aligned views of the
    same data takes its planned 4-byte fallback and matches the oracle."""
    fails = []
    for R, C in [(64, 1 << 16), (1 << 15, 64), (8192, 1024), (8, 1 << 18), (4096, 16), (256, 4096)]:
        M = synth.matrix(R, C, op, np.float32, "uniform", synth.seed(14, "A") + R)
        X = synth.matrix(K, C, "mv", np.float32, "uniform", synth.seed(14, "x") + C)
        for off in (1, 2, 3):
            Mb = torch.empty(M.size + off, dtype=torch.float32, device=DEV)
            Xb = torch.empty(X.size + off, dtype=torch.float32, device=DEV)
            Yb = torch.empty(K * R + off, dtype=torch.float32, device=DEV)
            Md = Mb[off:].view(M.shape)
            Xd = Xb[off:].view(X.shape)
            Md.copy_(torch.from_numpy(M))
            Xd.copy_(torch.from_numpy(X))
            Yd = Yb[off:].view(K, R)
            try:
                fn = adaptic.mv_multi if op == "mv" else adaptic.tmv_multi
                fn(Md, Xd, out=Yd)
                check(Yd.cpu().numpy(), M, X, op, f"{op} {R}x{C} K={K} off={off}")
            except Exception as e:  # noqa: BLE001
                fails.append(f"{op} {R}x{C} K={K} off={off}: {type(e).__name__}: {str(e)[:160]}")
    assert not fails, "\n".join(fails)


@pytest.mark.parametrize("K", [2, 4, 8])
def test_tmv_row_groups_of_four(K):
    """tmmv4_kernel (XSMEM 8): x_j read as one float4 per 4 rows, optional L2 prefetch; tiles,
    splits (ticket merge) and ragged tiles against the oracle."""
    fails = []
    for (R, C), p in itertools.product([(4, 4), (64, 4096), (1028, 1000), (8192, 64), (260, 40000), (4096, 1 << 16)],
                                       [[0, 0, 0, 0, 8], [16, 0, 0, 2, 8], [64, 7, 0, 4, 8], [256, 0, 0, 1, 8]]):
        B = synth.matrix(R, C, "tmv", np.float32, "uniform", synth.seed(15, "A") + R)
        X = synth.matrix(K, C, "mv", np.float32, "uniform", synth.seed(15, "x") + C)
        try:
            assert adaptic.plan("tmv", R, C, variant="TMV_SPLITK", params=p, nvec=K).describe()["xmode"] == 8
            Y = adaptic.tmv_multi(torch.from_numpy(B).to(DEV), torch.from_numpy(X).to(DEV), variant="TMV_SPLITK",
                                  params=p).cpu().numpy()
            check(Y, B, X, "tmv", f"tmmv4 {R}x{C} {p}")
        except Exception as e:  # noqa: BLE001
            fails.append(f"{R}x{C} {p}: {type(e).__name__}: {str(e)[:160]}")
    assert not fails, "\n".join(fails)
