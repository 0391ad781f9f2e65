"""BiCGSTAB oracle -- TEST INFRASTRUCTURE ONLY (same import rules as the package:
only tests/, __graft_entry__.smoke() and bench.py's CPU legs use it).

The paper's second case study (Sec. 5.2.2) is the biconjugate
gradient stabilized method for nonsymmetric Ax = b, "11 linear steps that can be
written easily with the CUBLAS library" (Sgemv, Sdot, Sscal, Saxpy).  The paper
does not print the steps; this is the textbook unpreconditioned method (van der
Vorst, 1992), written out in plain numpy fp64 in that order, with x0 = 0 and the
shadow residual r^ = r0 = b.  Matrix-vector products and dot products use numpy
primitives (np.dot / @) -- no blocking, no fusion:

  1  rho_i   = (r^, r_{i-1})
  2  beta    = (rho_i / rho_{i-1}) (alpha / omega)
  3  p_i     = r_{i-1} + beta (p_{i-1} - omega v_{i-1})
  4  v_i     = A p_i
  5  alpha   = rho_i / (r^, v_i)
  6  s       = r_{i-1} - alpha v_i
  7  (stop if ||s|| / ||b|| < tol: x_i = x_{i-1} + alpha p_i)
  8  t       = A s
  9  omega   = (t, s) / (t, t)
  10 x_i     = x_{i-1} + alpha p_i + omega s
  11 r_i     = s - omega t          (stop if ||r_i|| / ||b|| < tol)

with rho_0 = alpha = omega_0 = 1 and p_0 = v_0 = 0.  Pins: tests/test_oracle_bicgstab.py
(a 2x2 system solved by hand, A = I, diagonal A, LAPACK solve on random diagonally
dominant systems, the recurrence residual equal to b - A x).
"""
from __future__ import annotations

import numpy as np


def bicgstab(A: np.ndarray, b: np.ndarray, tol: float = 1e-6, max_iters: int = 1000):
    """Returns (x, iterations, history); history[i] = dict(rho, alpha, omega, relres)
    of iteration i+1 (omega is None when the iteration stopped at step 7)."""
    A = np.asarray(A, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    n = b.shape[0]
    x = np.zeros(n)
    r = b.copy()
    rhat = b.copy()
    p = np.zeros(n)
    v = np.zeros(n)
    rho_prev = alpha = omega = 1.0
    bnorm = float(np.sqrt(np.dot(b, b)))
    hist = []
    if bnorm == 0.0:
        return x, 0, hist
    for it in range(1, max_iters + 1):
        rho = float(np.dot(rhat, r))                                  # 1
        if rho == 0.0:
            break                                                     # breakdown
        beta = (rho / rho_prev) * (alpha / omega)                     # 2
        p = r + beta * (p - omega * v)                                # 3
        v = A @ p                                                     # 4
        alpha = rho / float(np.dot(rhat, v))                          # 5
        s = r - alpha * v                                             # 6
        snorm = float(np.sqrt(np.dot(s, s)))
        if snorm / bnorm < tol:                                       # 7
            x = x + alpha * p
            hist.append({"rho": rho, "alpha": alpha, "omega": None, "relres": snorm / bnorm})
            return x, it, hist
        t = A @ s                                                     # 8
        omega = float(np.dot(t, s)) / float(np.dot(t, t))             # 9
        x = x + alpha * p + omega * s                                 # 10
        r = s - omega * t                                             # 11
        rho_prev = rho
        relres = float(np.sqrt(np.dot(r, r))) / bnorm
        hist.append({"rho": rho, "alpha": alpha, "omega": omega, "relres": relres})
        if relres < tol:
            return x, it, hist
        if omega == 0.0:
            break
    return x, len(hist), hist
