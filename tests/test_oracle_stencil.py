"""Pins for the five-point stencil oracle (oracle_stencil5_f64; the paper's
neighbouring-access actor, Sec. 4.1.2, Fig. 4a; reading R19).
CPU only."""
import numpy as np
import pytest

import oracle
import synth


def test_3x3_by_hand():
    """Only the centre is interior: v[1][1] = c*5 + n*(2 + 8 + 4 + 6); the edge is copied."""
    u = np.arange(1, 10, dtype=np.float32).reshape(3, 3)     # [[1,2,3],[4,5,6],[7,8,9]]
    v, S = oracle.stencil5(u, 0.5, 0.125)
    expect = u.astype(np.float64).copy()
    expect[1, 1] = 0.5 * 5 + 0.125 * (2 + 8 + 4 + 6)           # = 5.0
    assert np.array_equal(v, expect)
    assert S[1, 1] == 0.5 * 5 + 0.125 * 20


def test_harmonic_fields_are_fixed_points():
    """With c + 4n = 1 the stencil is a weighted average; a discrete-harmonic field
    (constant, linear a*i + b*j, or i*j) is reproduced exactly at every point."""
    H, W = 17, 23
    i, j = np.meshgrid(np.arange(H), np.arange(W), indexing="ij")
    for field in (np.full((H, W), 3.0), 2.0 * i - 3.0 * j + 1.0, (i * j).astype(np.float64), i * i - j * j):
        u = field.astype(np.float32)
        v, _ = oracle.stencil5(u, 0.6, 0.1)
        assert np.allclose(v, u.astype(np.float64), rtol=0, atol=1e-12)


def test_against_numpy_slicing():
    """The same definition written with array slices (an independent formulation)."""
    u = synth.matrix(40, 57, "mv", np.float32, "uniform", 3)
    c, n = -1.25, 0.375
    v, _ = oracle.stencil5(u, c, n)
    ud = u.astype(np.float64)
    ref = ud.copy()
    ref[1:-1, 1:-1] = c * ud[1:-1, 1:-1] + n * (ud[:-2, 1:-1] + ud[2:, 1:-1] + ud[1:-1, :-2] + ud[1:-1, 2:])
    assert np.allclose(v, ref, rtol=0, atol=1e-14)


def test_transpose_symmetry_and_degenerate():
    u = synth.matrix(31, 12, "mv", np.float32, "uniform", 4)
    v, _ = oracle.stencil5(u, 0.3, 0.2)
    vt, _ = oracle.stencil5(np.ascontiguousarray(u.T), 0.3, 0.2)
    assert np.allclose(v.T, vt, rtol=0, atol=1e-14)
    for H, W in ((1, 5), (5, 1), (2, 2), (0, 3)):
        u = synth.matrix(max(H, 1), W, "mv", np.float32, "uniform", 5)[:H]
        v, _ = oracle.stencil5(u, 0.3, 0.2)
        assert np.array_equal(v, u.astype(np.float64))           # no interior point
