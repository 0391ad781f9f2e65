"""Pins for the BiCGSTAB oracle (oracle/bicgstab.py; the paper's Sec. 5.2.2 case
study).  CPU only."""
import numpy as np
import pytest

import synth
from oracle.bicgstab import bicgstab


def test_2x2_by_hand():
    """A = [[4, 1], [2, 3]], b = [1, 2]: x* = [0.1, 0.6] (Cramer: det 10, x1 = (3-2)/10,
    x2 = (8-2)/10).  A Krylov method on a 2x2 system is exact after at most 2 iterations."""
    x, it, _ = bicgstab(np.array([[4.0, 1.0], [2.0, 3.0]]), np.array([1.0, 2.0]), tol=1e-14)
    assert it <= 2
    assert np.allclose(x, [0.1, 0.6], rtol=0, atol=1e-14)


def test_identity_one_step():
    """A = I: p = r = b, v = b, alpha = 1, s = 0 -> stops at step 7 with x = b."""
    b = synth.vector(50, np.float32, "uniform", 3).astype(np.float64)
    x, it, hist = bicgstab(np.eye(50), b, tol=1e-12)
    assert it == 1 and hist[0]["alpha"] == 1.0 and hist[0]["omega"] is None
    assert np.array_equal(x, b)


def test_diagonal_system():
    d = np.arange(1, 41, dtype=np.float64)
    b = synth.vector(40, np.float32, "uniform", 4).astype(np.float64)
    x, it, _ = bicgstab(np.diag(d), b, tol=1e-13, max_iters=200)
    assert np.allclose(x, b / d, rtol=1e-11, atol=0)


@pytest.mark.parametrize("n", [16, 64, 200])
def test_diagonally_dominant_against_lapack(n):
    """The synthetic systems (synth 'diagdom': off-diagonal U[-1,1), diagonal n): the
    converged oracle solution equals LAPACK's direct solve, and its true residual
    meets the tolerance."""
    A = synth.matrix(n, n, "mv", np.float32, "diagdom", synth.seed(20, "A")).astype(np.float64)
    b = synth.vector(n, np.float32, "uniform", synth.seed(20, "b")).astype(np.float64)
    x, it, hist = bicgstab(A, b, tol=1e-12, max_iters=500)
    xs = np.linalg.solve(A, b)
    assert np.allclose(x, xs, rtol=0, atol=1e-10 * np.abs(xs).max())
    assert np.linalg.norm(b - A @ x) / np.linalg.norm(b) < 1e-11
    assert hist[-1]["relres"] < 1e-12 and it < 100


def test_recurrence_residual_is_true_residual():
    """r_i (step 11) = b - A x_i in exact arithmetic: a dropped or sign-flipped term in
    steps 3, 6, 10 or 11 breaks this identity."""
    n = 120
    A = synth.matrix(n, n, "mv", np.float32, "diagdom", 7).astype(np.float64)
    A += np.diag(np.linspace(-50, 50, n))              # less benign spectrum: more iterations
    b = synth.vector(n, np.float32, "uniform", 8).astype(np.float64)
    for k in range(1, 6):
        x, it, hist = bicgstab(A, b, tol=0.0, max_iters=k)
        assert it == k
        true = np.linalg.norm(b - A @ x) / np.linalg.norm(b)
        assert abs(true - hist[-1]["relres"]) <= 1e-12, (k, true, hist[-1]["relres"])


def test_nonsymmetric_needs_bicgstab_not_cg():
    """A rotation-like nonsymmetric system (skew part dominates): still solved."""
    n = 60
    rng_free = synth.matrix(n, n, "mv", np.float32, "uniform", 9).astype(np.float64)
    A = 4 * np.eye(n) + (rng_free - rng_free.T)          # I-shifted skew-symmetric
    b = synth.vector(n, np.float32, "uniform", 10).astype(np.float64)
    x, it, _ = bicgstab(A, b, tol=1e-12, max_iters=1000)
    assert np.allclose(A @ x, b, rtol=0, atol=1e-9)
