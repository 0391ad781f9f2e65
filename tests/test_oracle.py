"""Pins for the CPU oracle, run without a GPU.

Each test checks the oracle against something other than itself: values printed
in the paper or computed by hand (tests/golden/), closed forms, Python big-int
arithmetic, math.fsum (correctly rounded), numpy float64, brute-force
invariants.  A plausible slip in oracle.c -- a dropped term, a wrong index or
sign, a transposed operand, a missing wrap -- fails at least one of them:

  dropped / extra term ........ P1 ones, hand cases, fsum
  wrong index (r*R+c, c*C+r) .. hand cases (non-square), P6, perm
  transposed operand in TMV ... tmv hand case, P6 on non-square, Fig. 3 map
  sign ........................ hand case mv2, fsum on U[-1,1)
  int32 not wrapping / signed . big-int mod 2^32, int32_wrap golden
  S (magnitude) wrong ......... S >= |y|, S == y on non-negative data, fsum of |p|
"""
import json
import math
import os

import numpy as np
import pytest

import oracle
import synth

RNG = np.random.default_rng(1234)
U = 2.0 ** -53  # unit roundoff of the oracle's double accumulator


def _load(golden_dir, name):
    with open(os.path.join(golden_dir, name)) as f:
        return json.load(f)


# ---------------------------------------------------------------- hand cases (P11)
def test_hand_cases(golden_dir):
    g = _load(golden_dir, "hand_cases.json")
    for key in ("mv", "mv2"):
        A = np.array(g[key]["A"], np.float32)
        x = np.array(g[key]["x"], np.float32)
        y, S = oracle.mv(A, x)
        assert y.tolist() == g[key]["y"]
        yi = oracle.mv(A.astype(np.int32), x.astype(np.int32))
        assert yi.tolist() == g[key]["y"]
    B = np.array(g["tmv"]["B"], np.float32)
    x = np.array(g["tmv"]["x"], np.float32)
    y, _ = oracle.tmv(B, x)
    assert y.tolist() == g["tmv"]["y"]
    assert oracle.tmv(B.astype(np.int32), x.astype(np.int32)).tolist() == g["tmv"]["y"]
    a = np.array(g["dot"]["a"], np.float32)
    b = np.array(g["dot"]["b"], np.float32)
    y, _ = oracle.dot(a, b)
    assert y.tolist() == g["dot"]["y"]
    assert oracle.dot(a.astype(np.int32), b.astype(np.int32)).tolist() == g["dot"]["y"]


def test_int32_wrap_golden(golden_dir):
    g = _load(golden_dir, "hand_cases.json")["int32_wrap"]
    for case in g["cases"]:
        A = np.array(case["A"], np.int64).astype(np.int32)
        x = np.array(case["x"], np.int64).astype(np.int32)
        assert oracle.mv(A, x).tolist() == case["y"]
        assert oracle.tmv(np.ascontiguousarray(A.T), x).tolist() == case["y"]


# ---------------------------------------------------------------- Fig. 3 (P13)
def test_fig3_restructure_addresses(golden_dir):
    g = _load(golden_dir, "fig3_restructure.json")
    T, P = g["threads"], g["pops"]
    words = np.arange(T * P, dtype=np.float32)          # word w holds value w
    # before: thread t's k-th pop reads word P*t + k  (printed in the paper)
    before = words.reshape(T, P)
    assert before[:, 0].astype(int).tolist() == g["before_first_pop"]
    assert before[:3, 1].astype(int).tolist() == g["before_second_pop_head"]
    assert int(before[T - 1, 1]) == g["before_second_pop_last"]
    after = oracle.restructure(words, T, P)
    for k in range(P):
        # pop k of all threads now reads consecutive words 64k .. 64k+63 ...
        seg = after[T * k: T * (k + 1)]
        # ... and those words hold exactly what thread t popped at pop k before
        assert seg.astype(int).tolist() == before[:, k].astype(int).tolist()


def test_restructure_maps_mv_buffer_to_tmv_buffer():
    R, C = 5, 7
    A = RNG.standard_normal((R, C)).astype(np.float32)
    B = oracle.restructure(A.ravel(), R, C).reshape(C, R)
    assert np.array_equal(B, A.T)
    x = RNG.standard_normal(C).astype(np.float32)
    assert np.array_equal(oracle.tmv(B, x)[0], oracle.mv(A, x)[0])


# ---------------------------------------------------------------- closed forms
@pytest.mark.parametrize("R,C", [(1, 1), (3, 5), (17, 33), (64, 1025), (2, 1 << 16)])
def test_P1_all_ones(R, C):
    A = np.ones((R, C), np.float32)
    x = np.ones(C, np.float32)
    y, S = oracle.mv(A, x)
    assert np.all(y == C) and np.all(S == C)
    y, S = oracle.tmv(np.ones((C, R), np.float32), x)
    assert np.all(y == C)
    assert np.all(oracle.mv(A.astype(np.int32), x.astype(np.int32)) == C)
    assert np.all(oracle.dot(A, A)[0] == C)


def test_P1_ones_at_2pow24():
    C = 1 << 24
    x = np.ones(C, np.float32)
    y, _ = oracle.mv(np.ones((1, C), np.float32), x)
    assert y[0] == float(C)
    assert oracle.dot(np.ones((1, C), np.int32), np.ones((1, C), np.int32))[0] == C


@pytest.mark.parametrize("n", [1, 2, 7, 64, 129])
def test_P2_identity_and_perm(n):
    x = synth.vector(n, np.float32, "uniform", 77)
    I = synth.matrix(n, n, "mv", np.float32, "identity", 0)
    assert np.array_equal(oracle.mv(I, x)[0], x.astype(np.float64))
    P = synth.matrix(n, n, "mv", np.float32, "perm", 0)
    assert np.array_equal(oracle.mv(P, x)[0], x[::-1].astype(np.float64))
    Pt = synth.matrix(n, n, "tmv", np.float32, "perm", 0)
    assert np.array_equal(oracle.tmv(Pt, x)[0], x[::-1].astype(np.float64))


@pytest.mark.parametrize("n", [1, 9, 300])
def test_P3_diagonal(n):
    D = synth.matrix(n, n, "mv", np.float32, "diag", 5)
    x = synth.vector(n, np.float32, "uniform", 6)
    d = np.diag(D)
    assert np.array_equal(oracle.mv(D, x)[0], d.astype(np.float64) * x.astype(np.float64))


def test_P4_rank_one():
    R, C = 40, 333
    u = RNG.standard_normal(R).astype(np.float32)
    v = RNG.standard_normal(C).astype(np.float32)
    A = np.outer(u, v).astype(np.float32)  # rounded to fp32; compare against the rounded A
    x = RNG.standard_normal(C).astype(np.float32)
    y, S = oracle.mv(A, x)
    # exact (u v^T) x differs from fl32(u v^T) x by <= 2^-24 per entry
    ref = u.astype(np.float64) * float(np.dot(v.astype(np.float64), x.astype(np.float64)))
    assert np.all(np.abs(y - ref) <= 2 ** -23 * S + 1e-12)


# ---------------------------------------------------------------- library / textbook (P12)
@pytest.mark.parametrize("R,C", [(1, 1), (4, 3), (33, 65), (7, 1024), (3, 5000)])
def test_P12_fsum_and_numpy(R, C):
    s = synth.seed(0, "A")
    A = synth.matrix(R, C, "mv", np.float32, "uniform", s)
    x = synth.vector(C, np.float32, "uniform", synth.seed(0, "x"))
    y, S = oracle.mv(A, x)
    A64, x64 = A.astype(np.float64), x.astype(np.float64)
    for r in range(R):
        prods = [float(a) * float(b) for a, b in zip(A64[r], x64)]
        exact = math.fsum(prods)                 # correctly rounded sum of exact products
        mag = math.fsum(abs(p) for p in prods)
        assert abs(y[r] - exact) <= C * U * mag + 1e-300
        assert abs(S[r] - mag) <= C * U * mag + 1e-300
    assert np.allclose(y, A64 @ x64, rtol=0, atol=1e-12 * max(1.0, S.max()))
    # TMV and DOT through the same definition
    B = np.ascontiguousarray(A.T)
    yt, St = oracle.tmv(B, x)
    assert np.array_equal(yt, y) and np.array_equal(St, S)          # P6: identical order
    yd, Sd = oracle.dot(A, np.broadcast_to(x, (R, C)).copy())
    assert np.array_equal(yd, y) and np.array_equal(Sd, S)


@pytest.mark.parametrize("R,C", [(1, 1), (5, 9), (64, 257), (2, 4096)])
def test_P12_int32_bigint(R, C):
    A = synth.matrix(R, C, "mv", np.int32, "uniform", 11)
    x = synth.vector(C, np.int32, "uniform", 12)
    x[0] = np.int32(-2**31)  # exercise the extremes
    A[0, 0] = np.int32(2**31 - 1)
    y = oracle.mv(A, x)
    for r in range(R):
        exact = sum(int(a) * int(b) for a, b in zip(A[r].tolist(), x.tolist()))
        m = exact % (1 << 32)
        expect = m - (1 << 32) if m >= (1 << 31) else m
        assert int(y[r]) == expect
    assert np.array_equal(oracle.tmv(np.ascontiguousarray(A.T), x), y)


def test_int32_dot_wrap_long():
    L = 1 << 22
    a = synth.matrix(1, L, "mv", np.int32, "positive", 21)
    b = synth.matrix(1, L, "mv", np.int32, "positive", 22)
    exact = int(np.dot(a[0].astype(np.int64), b[0].astype(np.int64)))  # < 2^36: exact in int64
    assert exact >= (1 << 32)  # the sum does wrap
    m = exact % (1 << 32)
    expect = m - (1 << 32) if m >= (1 << 31) else m
    assert int(oracle.dot(a, b)[0]) == expect


# ---------------------------------------------------------------- P5 exact regime
@pytest.mark.parametrize("kind", ["smallint", "smallint4"])
def test_P5_integer_valued_fp32_is_exact(kind):
    R, C = 9, 20000
    A = synth.matrix(R, C, "mv", np.float32, kind, 3)
    x = synth.vector(C, np.float32, kind, 4)
    y, _ = oracle.mv(A, x)
    exact = A.astype(np.int64) @ x.astype(np.int64)
    assert np.array_equal(y, exact.astype(np.float64))
    yi = oracle.mv(A.astype(np.int32), x.astype(np.int32))
    assert np.array_equal(yi.astype(np.int64), exact)


# ---------------------------------------------------------------- invariants
def test_P6_tmv_equals_mv_of_transpose_nonsquare():
    for R, C in [(3, 8), (8, 3), (31, 257)]:
        A = synth.matrix(R, C, "mv", np.float32, "uniform", 1)
        B = synth.matrix(R, C, "tmv", np.float32, "uniform", 1)
        assert np.array_equal(B, A.T)
        x = synth.vector(C, np.float32, "uniform", 2)
        assert np.array_equal(oracle.tmv(B, x)[0], oracle.mv(A, x)[0])
        Ai = synth.matrix(R, C, "mv", np.int32, "uniform", 1)
        xi = synth.vector(C, np.int32, "uniform", 2)
        assert np.array_equal(oracle.tmv(np.ascontiguousarray(Ai.T), xi), oracle.mv(Ai, xi))


def test_P8_linearity():
    R, C = 13, 777
    A = synth.matrix(R, C, "mv", np.int32, "uniform", 31)
    x = synth.vector(C, np.int32, "uniform", 32)
    z = synth.vector(C, np.int32, "uniform", 33)
    al, be = 3, -7
    lhs = oracle.mv(A, (al * x.astype(np.int64) + be * z.astype(np.int64)).astype(np.int32))
    rhs = (al * oracle.mv(A, x).astype(np.int64) + be * oracle.mv(A, z).astype(np.int64))
    assert np.array_equal(lhs.astype(np.uint32), (rhs % (1 << 32)).astype(np.uint32))
    Af = synth.matrix(R, C, "mv", np.float32, "uniform", 31)
    # x, z on a 2^-10 grid so that w = 0.5 x - 0.25 z is exact in fp32
    xf = (np.round(synth.vector(C, np.float32, "uniform", 32) * 1024) / 1024).astype(np.float32)
    zf = (np.round(synth.vector(C, np.float32, "uniform", 33) * 1024) / 1024).astype(np.float32)
    w = (0.5 * xf.astype(np.float64) - 0.25 * zf.astype(np.float64)).astype(np.float32)
    assert np.array_equal(w.astype(np.float64), 0.5 * xf.astype(np.float64) - 0.25 * zf.astype(np.float64))
    yw, Sw = oracle.mv(Af, w)
    yx, Sx = oracle.mv(Af, xf)
    yz, Sz = oracle.mv(Af, zf)
    assert np.all(np.abs(yw - (0.5 * yx - 0.25 * yz)) <= 4 * C * U * (Sw + Sx + Sz))


def test_P9_column_split_additivity():
    R, C, k = 6, 1000, 377
    A = synth.matrix(R, C, "mv", np.int32, "uniform", 41)
    x = synth.vector(C, np.int32, "uniform", 42)
    full = oracle.mv(A, x).astype(np.uint32)
    left = oracle.mv(np.ascontiguousarray(A[:, :k]), x[:k]).astype(np.uint32)
    right = oracle.mv(np.ascontiguousarray(A[:, k:]), x[k:]).astype(np.uint32)
    assert np.array_equal(full, left + right)  # uint32 addition wraps mod 2^32


def test_P10_row_shards_concatenate():
    R, C = 101, 64
    A = synth.matrix(R, C, "mv", np.float32, "uniform", 51)
    x = synth.vector(C, np.float32, "uniform", 52)
    full = oracle.mv(A, x)[0]
    parts = [oracle.mv(synth.matrix(R, C, "mv", np.float32, "uniform", 51, rows=(a, b)), x)[0]
             for a, b in [(0, 40), (40, 41), (41, 101)]]
    assert np.array_equal(np.concatenate(parts), full)


def test_magnitude_S():
    R, C = 8, 500
    A = synth.matrix(R, C, "mv", np.float32, "uniform", 61)
    x = synth.vector(C, np.float32, "uniform", 62)
    y, S = oracle.mv(A, x)
    assert np.all(S >= np.abs(y))
    Ap = synth.matrix(R, C, "mv", np.float32, "positive", 61)
    xp = synth.vector(C, np.float32, "positive", 62)
    yp, Sp = oracle.mv(Ap, xp)
    assert np.array_equal(yp, Sp)


def test_rows_matches_full():
    R, C = 37, 91
    A = synth.matrix(R, C, "mv", np.float32, "uniform", 71)
    x = synth.vector(C, np.float32, "uniform", 72)
    y, S = oracle.mv(A, x)
    idx = [0, 5, 36, 17]
    yr, Sr = oracle.rows("mv", A, x, R, C, idx)
    assert np.array_equal(yr, y[idx]) and np.array_equal(Sr, S[idx])
    B = np.ascontiguousarray(A.T)
    yr, Sr = oracle.rows("tmv", B, x, R, C, idx)
    assert np.array_equal(yr, y[idx])
    Ai = synth.matrix(R, C, "mv", np.int32, "uniform", 71)
    xi = synth.vector(C, np.int32, "uniform", 72)
    assert np.array_equal(oracle.rows("tmv", np.ascontiguousarray(Ai.T), xi, R, C, idx),
                          oracle.mv(Ai, xi)[idx])


def test_nan_stays_in_its_row():
    R, C = 4, 10
    A = synth.matrix(R, C, "mv", np.float32, "uniform", 81)
    A[2, 3] = np.nan
    x = synth.vector(C, np.float32, "uniform", 82)
    y, _ = oracle.mv(A, x)
    assert np.isnan(y[2]) and not np.isnan(np.delete(y, 2)).any()


def test_degenerate_shapes():
    y, S = oracle.mv(np.zeros((0, 5), np.float32), np.zeros(5, np.float32))
    assert y.shape == (0,)
    y, S = oracle.mv(np.zeros((4, 0), np.float32), np.zeros(0, np.float32))
    assert np.array_equal(y, np.zeros(4)) and np.array_equal(S, np.zeros(4))
    yi = oracle.tmv(np.zeros((0, 3), np.int32), np.zeros(0, np.int32))
    assert np.array_equal(yi, np.zeros(3, np.int32))
