"""Misaligned-row MV/DOT kernels (C % 4 != 0: 128-bit body + scalar head/tail,
csrc/mv_mis_kernels.cuh) against the oracle -- needs a GPU.

fp32 within 1e-4 * S_r (north_star), int32 bit-exact.  Covers every head length
h = 0..3 (rows start at every alignment), every forced variant, base pointers that
are not 16-byte aligned, and DOT operands whose addresses differ modulo 16 (which
take the scalar kernels)."""
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
FORCED = [("AUTO", None)] + [("MV_SUBWARP", [g, 0, 0, u]) for g in (1, 4, 16) for u in (1, 2, 4, 8)] + \
         [("MV_WPR", [0, 0, 0, u, xm]) for u in (1, 2, 4, 8) for xm in (1, 2)] + \
         [("MV_CPR", [nt, 0, 0, u, xm]) for nt, u in ((256, 2), (256, 4), (256, 8), (1024, 2), (1024, 4))
          for xm in (1, 2)] + \
         [("MV_SPLIT", [nt, s, 0, u, 0, 0, 0, o]) for nt, u in ((256, 4), (1024, 2)) for s in (2, 5) for o in (1, 2)] + \
         [("MV_SUBWARP", [g, 0, 0, u, 5]) for g, u in ((1, 4), (4, 2), (16, 1))] + \
         [("MV_WPR", [0, 0, 0, u, 5]) for u in (1, 8)] + [("MV_CPR", [256, 0, 0, 4, 5]), ("MV_CPR", [1024, 0, 0, 2, 5])] + \
         [("MV_SPLIT", [256, s, 0, 4, 5, 0, 0, o]) for s in (2, 5) for o in (1, 2)]


def check(y, ref, dt, what):
    if dt == "i32":
        assert np.array_equal(y, ref), f"{what}: int32 mismatch at {np.nonzero(y != ref)[0][:8]}"
    else:
        yr, S = ref
        err = np.abs(y.astype(np.float64) - yr)
        bad = ~(err <= TOL * S)
        assert not bad.any(), f"{what}: {bad.sum()} out of tolerance, worst {np.max(err - TOL * S)}"


def _collect(cases):
    fails = []
    for what, fn in cases:
        try:
            fn()
        except Exception as e:  # noqa: BLE001 -- report every failing case at once
            fails.append(f"{what}: {type(e).__name__}: {str(e)[:200]}")
    assert not fails, f"{len(fails)} failures:\n" + "\n".join(fails[:40])


@pytest.mark.parametrize("op", ["mv", "dot"])
@pytest.mark.parametrize("dt", ["f32", "i32"])
def test_every_variant_every_head_length(op, dt):
    npdt = np.float32 if dt == "f32" else np.int32
    shapes = [(7, 17), (9, 18), (33, 19), (65, 127), (130, 1001), (3, 4099), (257, 66), (5, 100003), (1000, 21)]

    def case(R, C, v, p):
        A = synth.matrix(R, C, "mv", npdt, "uniform", synth.seed(11, "A") + R + C)
        X = (synth.matrix(R, C, "mv", npdt, "uniform", synth.seed(11, "b") + R) if op == "dot"
             else synth.vector(C, npdt, "uniform", synth.seed(11, "x") + C))
        try:
            plan = adaptic.plan(op, R, C, dt, variant=v, params=p)
        except adaptic.AdapticError as e:
            assert e.status == L.ERR_UNSUPPORTED, str(e)
            return
        if C >= 16 and v != "AUTO":
            assert plan.describe()["mis"], plan.describe()
        fn = adaptic.mv if op == "mv" else adaptic.dot
        y = fn(torch.from_numpy(A).to(DEV), torch.from_numpy(X).to(DEV), variant=v, params=p).cpu().numpy()
        ref = oracle.mv(A, X) if op == "mv" else oracle.dot(A, X)
        check(y, ref, dt, f"{op} {dt} {R}x{C} {v} {p}")
    _collect([(f"{R}x{C} {v} {p}", lambda R=R, C=C, v=v, p=p: case(R, C, v, p))
              for (R, C), (v, p) in itertools.product(shapes, FORCED)])


def test_unaligned_base_pointer_any_C():
    """The head length is computed from the actual row address, so a matrix whose
    base is only 4-byte aligned runs the same kernels."""
    for R, C, off in [(31, 37, 1), (64, 1001, 2), (9, 5000, 3), (100, 16, 1)]:
        A = synth.matrix(R, C, "mv", np.float32, "uniform", 5 + C)
        x = synth.vector(C, np.float32, "uniform", 6 + C)
        big = torch.zeros(R * C + 8, dtype=torch.float32, device=DEV)
        big[off:off + R * C] = torch.from_numpy(A.reshape(-1)).to(DEV)
        Ad = big[off:off + R * C].view(R, C)
        for v in ("AUTO", "MV_SUBWARP", "MV_WPR", "MV_CPR", "MV_SPLIT"):
            try:
                y = adaptic.mv(Ad, torch.from_numpy(x).to(DEV), variant=v).cpu().numpy()
            except adaptic.AdapticError as e:
                assert e.status == L.ERR_UNSUPPORTED
                continue
            check(y, oracle.mv(A, x), "f32", f"off {off} {R}x{C} {v}")


def test_dot_operands_with_different_alignment():
    """a and b differing modulo 16 bytes: the scalar kernels (still exact/in tolerance)."""
    R, C = 17, 1003
    a = synth.matrix(R, C, "mv", np.int32, "uniform", 71)
    b = synth.matrix(R, C, "mv", np.int32, "uniform", 72)
    bb = torch.zeros(R * C + 4, dtype=torch.int32, device=DEV)
    bb[1:1 + R * C] = torch.from_numpy(b.reshape(-1)).to(DEV)
    for v in ("AUTO", "MV_WPR", "MV_CPR", "MV_SPLIT"):
        y = adaptic.dot(torch.from_numpy(a).to(DEV), bb[1:1 + R * C].view(R, C), variant=v).cpu().numpy()
        check(y, oracle.dot(a, b), "i32", f"dot mismatched {v}")


@pytest.mark.parametrize("k", [2, 5, 8, 11, 14, 17, 20])
def test_held_out_shapes_3x2k(k):
    """The selector's held-out grid (SURVEY 8(d) configs[1]): R = 3*2^k, C = 2^26/R
    (not a multiple of 4), scaled to 2^22 elements for the oracle, exact on smallint."""
    R = 3 << (k - 2) if k >= 2 else 3
    C = (1 << 22) // R
    for kind, dt in (("uniform", "f32"), ("smallint", "f32"), ("uniform", "i32")):
        npdt = np.float32 if dt == "f32" else np.int32
        A = synth.matrix(R, C, "mv", npdt, kind, synth.seed(1, "A"))
        x = synth.vector(C, npdt, kind, synth.seed(1, "x"))
        y = adaptic.mv(torch.from_numpy(A).to(DEV), torch.from_numpy(x).to(DEV)).cpu().numpy()
        ref = oracle.mv(A, x)
        if kind == "smallint" and dt == "f32":
            assert np.array_equal(y.astype(np.float64), ref[0]), f"P5 exact {R}x{C}"
        else:
            check(y, ref, dt, f"held-out {R}x{C} {kind} {dt}")


TMV_FORCED = [("AUTO", None), ("TMV_COL", [0, 0, 0, 4]), ("TMV_COL", [0, 0, 0, 8])] + \
             [("TMV_SPLITK", [lr, s, 0, u]) for lr in (1, 4, 32, 256) for s in (0, 3) for u in (2, 8)] + \
             [("TMV_REGTILE", [0, 0, 0, u]) for u in (2, 4)]


@pytest.mark.parametrize("dt", ["f32", "i32"])
def test_tmv_misaligned_rows_every_variant(dt):
    """R % 4 != 0: B's rows start at every alignment; two aligned loads + funnel shift."""
    npdt = np.float32 if dt == "f32" else np.int32
    shapes = [(9, 33), (13, 1000), (63, 257), (129, 4099), (1023, 65), (5, 100003), (1001, 1001), (30, 7),
              (1, 1000), (2, 77), (3, 100000), (1, 1), (7, 3), (62, 1 << 16)]

    def case(R, C, v, p):
        B = synth.matrix(R, C, "tmv", npdt, "uniform", synth.seed(12, "A") + R + C)
        x = synth.vector(C, npdt, "uniform", synth.seed(12, "x") + C)
        try:
            y = adaptic.tmv(torch.from_numpy(B).to(DEV), torch.from_numpy(x).to(DEV), variant=v, params=p)
        except adaptic.AdapticError as e:
            assert e.status == L.ERR_UNSUPPORTED, str(e)
            return
        check(y.cpu().numpy(), oracle.tmv(B, x), dt, f"tmv {dt} {R}x{C} {v} {p}")
    _collect([(f"{R}x{C} {v} {p}", lambda R=R, C=C, v=v, p=p: case(R, C, v, p))
              for (R, C), (v, p) in itertools.product(shapes, TMV_FORCED)])


def test_tmv_misaligned_base_and_output():
    """B and y at every 4-byte offset (the kernel computes B's own offset b0)."""
    for R, C in [(9, 1000), (61, 333), (1027, 64)]:
        B = synth.matrix(R, C, "tmv", np.float32, "uniform", 91 + R)
        x = synth.vector(C, np.float32, "uniform", 92 + C)
        for off in (1, 2, 3):
            big = torch.zeros(R * C + 8, dtype=torch.float32, device=DEV)
            big[off:off + R * C] = torch.from_numpy(B.reshape(-1)).to(DEV)
            yb = torch.zeros(R + 8, dtype=torch.float32, device=DEV)
            for v in ("AUTO", "TMV_COL", "TMV_SPLITK", "TMV_REGTILE"):
                try:
                    adaptic.tmv(big[off:off + R * C].view(C, R), torch.from_numpy(x).to(DEV), variant=v,
                                out=yb[off:off + R])
                except adaptic.AdapticError as e:
                    assert e.status == L.ERR_UNSUPPORTED
                    continue
                check(yb[off:off + R].cpu().numpy(), oracle.tmv(B, x), "f32", f"tmv off {off} {R}x{C} {v}")


@pytest.mark.parametrize("dt", ["f32", "i32"])
def test_tpr_rows_off_the_16_byte_grid(dt):
    """MV_TPR with C % 4 != 0: tiles are still 16-byte-granular bulk copies (the last,
    partial tile's remainder by plain loads), rows read as 32-bit words."""
    npdt = np.float32 if dt == "f32" else np.int32
    for R, C in [(1, 5), (3, 17), (255, 9), (256, 13), (1000, 65), (4097, 33), (100003, 7), (777, 2)]:
        for op in ("mv", "dot"):
            A = synth.matrix(R, C, "mv", npdt, "uniform", 31 + R + C)
            X = (synth.matrix(R, C, "mv", npdt, "uniform", 32 + R) if op == "dot"
                 else synth.vector(C, npdt, "uniform", 33 + C))
            for p in (None, [128, 0, 0, 2], [256, 0, 0, 4]):
                try:
                    plan = adaptic.plan(op, R, C, dt, variant="MV_TPR", params=p)
                except adaptic.AdapticError as e:
                    assert e.status == L.ERR_UNSUPPORTED
                    continue
                assert plan.describe()["mis"]
                fn = adaptic.mv if op == "mv" else adaptic.dot
                y = fn(torch.from_numpy(A).to(DEV), torch.from_numpy(X).to(DEV), variant="MV_TPR", params=p)
                ref = oracle.mv(A, X) if op == "mv" else oracle.dot(A, X)
                check(y.cpu().numpy(), ref, dt, f"tpr {op} {dt} {R}x{C} {p}")


def test_shifted_x_copies_any_x_alignment():
    """[ADAPTIC_P_XSMEM] = 5 (misaligned MV rows): x is first copied into four shifted,
    16-byte-aligned copies in the workspace, so x may sit at any 4-byte offset."""
    for R, C in [(37, 1001), (5, 100003), (3000, 77)]:
        A = synth.matrix(R, C, "mv", np.float32, "uniform", 61 + C)
        x = synth.vector(C, np.float32, "uniform", 62 + C)
        Ad = torch.from_numpy(A).to(DEV)
        for off in (0, 1, 2, 3):
            xb = torch.zeros(C + 8, dtype=torch.float32, device=DEV)
            xb[off:off + C] = torch.from_numpy(x).to(DEV)
            for v, p in (("MV_WPR", [0, 0, 0, 2, 5]), ("MV_CPR", [256, 0, 0, 4, 5]),
                         ("MV_SPLIT", [256, 3, 0, 4, 5])):
                y = adaptic.mv(Ad, xb[off:off + C], variant=v, params=p).cpu().numpy()
                check(y, oracle.mv(A, x), "f32", f"shift x off {off} {R}x{C} {v}")


def test_shifted_x_row_groups_share_x():
    """mv_cta_mis_rb_kernel (MV_SPLIT / MV_CPR, XSMEM 5, ROWS 2 or 4): RB rows of one residue
    class (r mod 4: same head, same shifted copy of x) per CTA step; ragged groups (R not a
    multiple of 4 RB), splits (ticket merge per group), every base alignment; fp32 within
    1e-4 S_r, int32 exact."""
    import itertools
    fails = []
    for (R, C), off, p in itertools.product([(1, 1001), (7, 40001), (64, 65537), (130, 3003), (517, 1025)],
                                            (0, 1, 3),
                                            [[256, 0, 0, 4, 5, 0, 2], [256, 0, 0, 2, 5, 0, 4], [256, 5, 0, 4, 5, 0, 4, 1],
                                             [256, 0, 0, 2, 5, 0, 2, 2]]):
        for dt in ("f32", "i32"):
            np_dt = np.float32 if dt == "f32" else np.int32
            tdt = torch.float32 if dt == "f32" else torch.int32
            A = synth.matrix(R, C, "mv", np_dt, "uniform", 31 + R)
            x = synth.vector(C, np_dt, "uniform", 32 + C)
            buf = torch.zeros(A.size + 8, dtype=tdt, device=DEV)
            buf[off:off + A.size] = torch.from_numpy(A.reshape(-1)).to(DEV)
            try:
                for v in ("MV_SPLIT", "MV_CPR"):
                    d = adaptic.plan("mv", R, C, dt, variant=v, params=p).describe()
                    assert d["xmode"] == 3, d
                    y = adaptic.mv(buf[off:off + A.size].view(R, C), torch.from_numpy(x).to(DEV), variant=v,
                                   params=p).cpu().numpy()
                    if dt == "i32":
                        assert np.array_equal(y, oracle.mv(A, x)), "int32 mismatch"
                    else:
                        yr, S = oracle.mv(A, x)
                        assert np.all(np.abs(y.astype(np.float64) - yr) <= 1e-4 * S), "out of tolerance"
            except Exception as e:  # noqa: BLE001
                fails.append(f"{dt} {R}x{C} off={off} {p}: {type(e).__name__}: {str(e)[:160]}")
    assert not fails, f"{len(fails)} failures\n" + "\n".join(fails[:20])


def test_x_funnel_cta_kernel():
    """mv_cta_mis_fx_kernel (MV_SPLIT / MV_CPR, XSMEM 9): x as two aligned 128-bit loads and a
    compile-time funnel per row head h = 0..3 (every row residue), the last body vector's
    x read word by word at the end of x; splits; x only 4-byte aligned -> the XM_LDG kernel."""
    import itertools
    fails = []
    for (R, C), off, xoff, p in itertools.product([(1, 1001), (7, 40001), (64, 65537), (130, 3003), (9, 1030)],
                                                  (0, 1, 3), (0, 1),
                                                  [[256, 0, 0, 4, 9], [256, 6, 0, 2, 9, 0, 0, 1], [256, 0, 0, 8, 9]]):
        for dt in ("f32", "i32"):
            np_dt = np.float32 if dt == "f32" else np.int32
            tdt = torch.float32 if dt == "f32" else torch.int32
            A = synth.matrix(R, C, "mv", np_dt, "uniform", 41 + R)
            x = synth.vector(C, np_dt, "uniform", 42 + C)
            buf = torch.zeros(A.size + 8, dtype=tdt, device=DEV)
            buf[off:off + A.size] = torch.from_numpy(A.reshape(-1)).to(DEV)
            xb = torch.zeros(C + 8, dtype=tdt, device=DEV)
            xb[xoff:xoff + C] = torch.from_numpy(x).to(DEV)
            try:
                for v in ("MV_SPLIT", "MV_CPR"):
                    y = adaptic.mv(buf[off:off + A.size].view(R, C), xb[xoff:xoff + C], variant=v,
                                   params=p).cpu().numpy()
                    if dt == "i32":
                        assert np.array_equal(y, oracle.mv(A, x)), "int32 mismatch"
                    else:
                        yr, S = oracle.mv(A, x)
                        assert np.all(np.abs(y.astype(np.float64) - yr) <= 1e-4 * S), "out of tolerance"
            except Exception as e:  # noqa: BLE001
                fails.append(f"{dt} {R}x{C} off={off} xoff={xoff} {p}: {type(e).__name__}: {str(e)[:160]}")
    assert not fails, f"{len(fails)} failures\n" + "\n".join(fails[:20])
