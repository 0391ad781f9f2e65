"""Pins for the BLAS-1 oracle functions (the paper's Fig. 9
CUBLAS benchmarks Sasum, Snrm2, Isamax/Isamin).  CPU only."""
import json
import math
import os

import numpy as np
import pytest

import oracle
import synth


def _golden(golden_dir):
    with open(os.path.join(golden_dir, "blas1_hand.json")) as f:
        return json.load(f)


def test_hand_cases(golden_dir):
    g = _golden(golden_dir)
    for c in g["asum"]:
        assert oracle.asum(np.array(c["x"], np.float32))[0] == c["y"]
    for c in g["nrm2"]:
        assert oracle.nrm2(np.array(c["x"], np.float32))[0][0] == c["y"]
    for c in g["iamax"]:
        assert oracle.iamax(np.array(c["x"], np.float32))[0] == c["y"]
    for c in g["iamin"]:
        assert oracle.iamin(np.array(c["x"], np.float32))[0] == c["y"]


def test_empty_rows():
    assert oracle.iamax(np.zeros((3, 0), np.float32)).tolist() == [0, 0, 0]
    assert oracle.asum(np.zeros((2, 0), np.float32)).tolist() == [0.0, 0.0]


@pytest.mark.parametrize("N,L", [(1, 1), (3, 1000), (7, 4099)])
def test_against_fsum_and_numpy(N, L):
    a = synth.matrix(N, L, "mv", np.float32, "uniform", 5)
    ya = oracle.asum(a)
    yn, ssq = oracle.nrm2(a)
    for n in range(N):
        row = [float(v) for v in a[n]]
        exact_abs = math.fsum(abs(v) for v in row)
        exact_sq = math.fsum(v * v for v in row)
        assert abs(ya[n] - exact_abs) <= L * 2.0 ** -53 * exact_abs
        assert abs(ssq[n] - exact_sq) <= L * 2.0 ** -53 * exact_sq
        assert abs(yn[n] - math.sqrt(exact_sq)) <= 4 * L * 2.0 ** -53 * math.sqrt(exact_sq)
    assert np.allclose(yn, np.linalg.norm(a.astype(np.float64), axis=1), rtol=1e-12, atol=0)
    # iamax / iamin: numpy argmax/argmin return the FIRST occurrence -> the BLAS rule
    assert np.array_equal(oracle.iamax(a), np.argmax(np.abs(a), axis=1) + 1)
    assert np.array_equal(oracle.iamin(a), np.argmin(np.abs(a), axis=1) + 1)


def test_ties_keep_first_index():
    a = np.array([[2, -5, 5, 1, -5], [0, 3, 0, -3, 0]], np.float32)
    assert oracle.iamax(a).tolist() == [2, 2]
    assert oracle.iamin(a).tolist() == [4, 1]


def test_relations_to_dot():
    """asum(a) = dot(|a|, 1) and nrm2(a)^2 = dot(a, a): the same reduction engine."""
    a = synth.matrix(4, 3000, "mv", np.float32, "uniform", 9)
    ones = np.ones_like(a)
    assert np.array_equal(oracle.asum(a), oracle.dot(np.abs(a), ones)[0])
    assert np.array_equal(oracle.nrm2(a)[1], oracle.dot(a, a)[0])
