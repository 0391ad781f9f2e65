"""Parity of the BLAS-1 reductions (ASUM / NRM2 / IAMAX / IAMIN; SURVEY 8(f) rank 1,
the paper's Fig. 9 CUBLAS benchmarks) through the C ABI against the CPU
oracle -- needs a GPU.

Tolerances (BLAS-1 readings):
  asum : |y - y_ref| <= 1e-4 * y_ref        (y_ref = sum |a| is its own S_r)
  nrm2 : |y - y_ref| <= 2^-23 * y_ref       (fp64 sum of exact squares, one rounding
                                             to fp32: at most one fp32 ulp)
  iamax/iamin : bit-exact (the comparison of |a| is exact)
"""
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
OPS = ("asum", "nrm2", "iamax", "iamin")
SIZES_R = [1, 2, 3, 5, 8, 17, 33, 64, 129, 257, 1025]
SIZES_C = [1, 2, 3, 4, 5, 7, 8, 9, 15, 16, 17, 31, 32, 33, 63, 64, 65, 127, 128, 129,
           255, 256, 257, 1023, 1024, 1025, 4099]
# forced variants with parameter overrides (ADAPTIC_NPARAMS layout, _lib.P_*)
FORCED = [("MV_SUBWARP", [g, 0, 0, 0, 0, 0, rb]) for g in (1, 2, 4, 8, 16) for rb in (1, 4)] + \
         [("MV_WPR", [0, 0, 0, 0, 0, 0, rb]) for rb in (1, 4)] + \
         [("MV_CPR", None)] + [("MV_SPLIT", [0, s]) for s in (2, 3, 7)] + [("MV_SPLIT", None)]


def ref(op, a):
    if op == "asum":
        return oracle.asum(a)
    if op == "nrm2":
        return oracle.nrm2(a)[0]
    return oracle.iamax(a) if op == "iamax" else oracle.iamin(a)


def gpu(op, a, variant="AUTO", params=None, dev_tensor=None):
    t = dev_tensor if dev_tensor is not None else torch.from_numpy(np.ascontiguousarray(a)).to(DEV)
    return getattr(adaptic, op)(t, variant=variant, params=params).cpu().numpy()


def check(op, y, yr, what):
    if op in ("iamax", "iamin"):
        bad = y.astype(np.int64) != yr
        assert not bad.any(), f"{what}: index mismatch rows {np.nonzero(bad)[0][:8]}: {y[bad][:4]} vs {yr[bad][:4]}"
        return
    err = np.abs(y.astype(np.float64) - yr)
    tol = (1e-4 if op == "asum" else 2.0 ** -23) * np.abs(yr)
    bad = ~(err <= tol)
    assert not bad.any(), f"{what}: {bad.sum()} out of tolerance, worst excess {np.max(err - tol)}"


def _collect(cases):
    fails = []
    for what, fn in cases:
        try:
            fn()
        except Exception as e:  # noqa: BLE001 -- report every failing case at once
            fails.append(f"{what}: {type(e).__name__}: {str(e)[:200]}")
    assert not fails, f"{len(fails)} failures:\n" + "\n".join(fails[:40])


@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("kind", ["uniform", "smallint"])
def test_bruteforce_auto(op, kind):
    def case(R, C):
        a = synth.matrix(R, C, "mv", np.float32, kind, synth.seed(5, "A") + R * 7919 + C)
        check(op, gpu(op, a), ref(op, a), f"{op} {kind} {R}x{C} AUTO")
    _collect([(f"{R}x{C}", lambda R=R, C=C: case(R, C)) for R, C in itertools.product(SIZES_R, SIZES_C)])


@pytest.mark.parametrize("op", OPS)
def test_every_forced_variant(op):
    """Every thread shape and split count on ragged shapes; smallint data has many
    ties in |a|, which pins the first-index rule of IAMAX/IAMIN on every variant."""
    shapes = [(1, 1), (3, 5), (7, 33), (33, 257), (129, 1025), (5, 4099), (1, 100003), (1000, 12)]

    def case(R, C, kind, v, p):
        a = synth.matrix(R, C, "mv", np.float32, kind, synth.seed(6, "A") + R + C)
        try:
            y = gpu(op, a, v, p)
        except adaptic.AdapticError as e:
            assert e.status == L.ERR_UNSUPPORTED, str(e)
            return
        check(op, y, ref(op, a), f"{op} {kind} {R}x{C} {v} {p}")
    _collect([(f"{R}x{C} {k} {v} {p}", lambda R=R, C=C, k=k, v=v, p=p: case(R, C, k, v, p))
              for (R, C), k, (v, p) in itertools.product(shapes, ["uniform", "smallint"], FORCED)])


def test_nrm2_no_overflow_or_underflow():
    """Squares of 1e30 overflow fp32 and of 1e-30 underflow it; the fp64 sum of exact
    squares does neither: nrm2([3e30, 4e30]) = 5e30, nrm2([3e-30, 4e-30]) = 5e-30."""
    for v in ("MV_SUBWARP", "MV_WPR", "MV_CPR", "MV_SPLIT"):
        for s in (1e30, 1e-30, 1e19, 1e-19):
            a = np.zeros((3, 1000), np.float32)
            a[:, 10] = np.float32(3 * s)
            a[:, 700] = np.float32(4 * s)
            check("nrm2", gpu("nrm2", a, v), ref("nrm2", a), f"nrm2 scale {s} {v}")
            assert np.isfinite(gpu("nrm2", a, v)).all()


def test_iamax_nan_inf_zero_rules():
    """BLAS rule: the running extreme starts at |a_1| and a NaN never compares
    greater/smaller, so only a leading NaN yields 1; +-inf is an ordinary maximum."""
    rows = [
        [np.nan, 1, 5, 2],         # leading NaN -> 1 (both)
        [1, np.nan, 5, 2],         # NaN skipped -> iamax 3, iamin 1
        [0, np.nan, np.nan, 0],    # -> iamax 1, iamin 1
        [2, -np.inf, np.inf, 3],   # -> iamax 2 (first inf), iamin 1
        [-0.0, 0.0, 1, -1],        # -> iamax 3, iamin 1 (|-0| = |0|)
        [7, 7, 7, 7],              # ties -> 1
        [1, 2, np.nan, -2],        # -> iamax 2, iamin 1
    ]
    a = np.array(rows, np.float32)
    big = np.tile(a, (1, 300))     # same pattern repeated: long rows, ties across splits
    for v in ("AUTO", "MV_SUBWARP", "MV_WPR", "MV_CPR", "MV_SPLIT"):
        for m in (a, big, np.ascontiguousarray(big[:, 1:])):
            for op in ("iamax", "iamin"):
                check(op, gpu(op, m, v), ref(op, m), f"{op} special {m.shape} {v}")


def test_asum_nrm2_nan_propagates_to_its_row():
    a = synth.matrix(6, 5000, "mv", np.float32, "uniform", 77)
    a[2, 4321] = np.nan
    for op in ("asum", "nrm2"):
        for v in ("MV_WPR", "MV_CPR", "MV_SPLIT"):
            y = gpu(op, a, v)
            assert np.isnan(y[2]) and np.isfinite(np.delete(y, 2)).all(), f"{op} {v}"


def test_positive_long_rows_asum_tolerance():
    """asum on U[0,1) data: a serial fp32 chain of 2^24 terms would break 1e-4; the
    planner's fold + split bound keeps every variant inside it."""
    a = synth.matrix(2, 1 << 24, "mv", np.float32, "positive", 11)
    for v in ("AUTO", "MV_WPR", "MV_CPR", "MV_SPLIT"):
        try:
            y = gpu("asum", a, v)
        except adaptic.AdapticError as e:
            assert e.status == L.ERR_UNSUPPORTED
            continue
        check("asum", y, ref("asum", a), f"asum positive {v}")


def test_misaligned_pointer_scalar_path():
    R, C = 9, 1001
    a = synth.matrix(R, C + 1, "mv", np.float32, "uniform", 3)
    t = torch.from_numpy(a).to(DEV).view(-1)[1:1 + R * C].view(R, C)   # 4-byte, not 16-byte aligned
    host = np.ascontiguousarray(a.reshape(-1)[1:1 + R * C].reshape(R, C))
    for op in OPS:
        for v in ("AUTO", "MV_SUBWARP", "MV_WPR", "MV_CPR", "MV_SPLIT"):
            check(op, gpu(op, None, v, dev_tensor=t), ref(op, host), f"{op} misaligned {v}")


def test_degenerate_and_errors():
    assert adaptic.asum(torch.empty(0, 5, device=DEV)).numel() == 0
    assert adaptic.iamax(torch.empty(4, 0, device=DEV)).cpu().tolist() == [0, 0, 0, 0]
    assert adaptic.nrm2(torch.empty(3, 0, device=DEV)).cpu().tolist() == [0.0, 0.0, 0.0]
    with pytest.raises(adaptic.AdapticError):
        adaptic.plan("asum", 4, 4, "i32")                  # fp32 only
    with pytest.raises(adaptic.AdapticError):
        adaptic.plan("iamax", 4, 4, variant="MV_TPR")
    with pytest.raises(adaptic.AdapticError):
        adaptic.plan("nrm2", 4, 4, variant="TMV_COL")


def test_rerun_identical_and_workspace_rearmed():
    a = torch.from_numpy(synth.matrix(3, 1 << 20, "mv", np.float32, "uniform", 21)).to(DEV)
    for op in OPS:
        y0 = getattr(adaptic, op)(a, variant="MV_SPLIT").cpu().numpy()
        for _ in range(3):
            assert np.array_equal(getattr(adaptic, op)(a, variant="MV_SPLIT").cpu().numpy(), y0), op


@pytest.mark.parametrize("k", [10, 16, 20, 24, 26, 27])
def test_single_vector_lengths(k):
    """Fig. 9's single-vector CUBLAS calls (n = 1K ... 4M) extended to
    B200 sizes: N = 1, L = 2^k, full comparison with the oracle."""
    a = synth.matrix(1, 1 << k, "mv", np.float32, "uniform", synth.seed(2, "A"))
    t = torch.from_numpy(a).to(DEV)
    for op in OPS:
        check(op, gpu(op, None, dev_tensor=t), ref(op, a), f"{op} N=1 L=2^{k}")


def test_device_generated_256MiB_batch():
    """The bench's BLAS-1 shapes (256 MiB, generated on the device): every output of
    a 64 x 2^20 batch against the oracle."""
    R, C = 64, 1 << 20
    t = torch.empty(R * C, dtype=torch.float32, device=DEV)
    synth.device_matrix(t, R, C, "mv", "uniform", synth.seed(7, "A"))
    a = t.cpu().numpy().reshape(R, C)
    t = t.view(R, C)
    for op in OPS:
        check(op, gpu(op, None, dev_tensor=t), ref(op, a), f"{op} 64x2^20")


# ------------------------------------------------------------------ horizontal actor integration
def check_all(a, outs, what):
    for op, y in zip(OPS, outs):
        check(op, y.cpu().numpy(), ref(op, a), f"b1all/{op} {what}")


@pytest.mark.parametrize("kind", ["uniform", "smallint"])
def test_b1all_matches_the_four_oracles(kind):
    """One pass computes asum, nrm2, iamax, iamin -- each equal to its own
    oracle (same tolerances / bit-exactness as the separate ops), every variant."""
    shapes = [(1, 1), (3, 5), (7, 33), (33, 257), (129, 1025), (5, 4099), (1, 100003), (1000, 12), (2, 1 << 20)]

    def case(R, C, v, p):
        a = synth.matrix(R, C, "mv", np.float32, kind, synth.seed(8, "A") + R + C)
        try:
            outs = adaptic.b1all(torch.from_numpy(a).to(DEV), variant=v, params=p)
        except adaptic.AdapticError as e:
            assert e.status == L.ERR_UNSUPPORTED, str(e)
            return
        check_all(a, outs, f"{kind} {R}x{C} {v} {p}")
    _collect([(f"{R}x{C} {v} {p}", lambda R=R, C=C, v=v, p=p: case(R, C, v, p))
              for (R, C), (v, p) in itertools.product(shapes, [("AUTO", None)] + FORCED)])


def test_b1all_special_values_and_degenerate():
    rows = [[np.nan, 1, 5, 2], [1, np.nan, 5, 2], [2, -np.inf, np.inf, 3], [7, 7, 7, 7], [0, 0, 0, 0]]
    a = np.tile(np.array(rows, np.float32), (1, 257))
    for v in ("AUTO", "MV_SUBWARP", "MV_WPR", "MV_CPR", "MV_SPLIT"):
        asum, nrm2, imax, imin = adaptic.b1all(torch.from_numpy(a).to(DEV), variant=v)
        check("iamax", imax.cpu().numpy(), ref("iamax", a), f"b1all special {v}")
        check("iamin", imin.cpu().numpy(), ref("iamin", a), f"b1all special {v}")
        assert np.isnan(asum.cpu().numpy()[:2]).all() and np.isinf(nrm2.cpu().numpy()[2])
    outs = adaptic.b1all(torch.empty(3, 0, device=DEV))
    assert all(o.cpu().tolist() == [0, 0, 0] for o in outs)


def test_b1all_256MiB_batch_and_single_vector():
    for R, C in [(64, 1 << 20), (1, 1 << 26)]:
        t = torch.empty(R * C, dtype=torch.float32, device=DEV)
        synth.device_matrix(t, R, C, "mv", "uniform", synth.seed(9, "A"))
        a = t.cpu().numpy().reshape(R, C)
        check_all(a, adaptic.b1all(t.view(R, C)), f"{R}x{C}")
