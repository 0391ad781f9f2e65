"""The shared input generator: vectorised numpy vs a pure-Python scalar splitmix64."""
import numpy as np
import pytest

import synth


def test_splitmix64_known_vector():
    # splitmix64 sequence from state 0 (first output of the public reference generator)
    assert synth.splitmix64_scalar(0) == 0xE220A8397B1DCDAF


@pytest.mark.parametrize("s", [0, 20120611, 2**63 + 5])
def test_hash_vectorised_matches_scalar(s):
    idx = np.array([0, 1, 2, 3, 12345, 2**32 + 7, 2**40 - 1], dtype=np.uint64)
    h = synth.hash64(s, idx)
    for i, v in zip(idx.tolist(), h.tolist()):
        assert v == synth.hash_scalar(s, i)


def test_value_ranges():
    s = synth.seed(1, "A")
    a = synth.vector(1 << 16, np.float32, "uniform", s)
    assert a.min() >= -1.0 and a.max() < 1.0 and abs(a.mean()) < 0.02
    assert np.all(a * 2.0**23 == np.round(a * 2.0**23))       # on the 2^-23 grid
    p = synth.vector(1 << 16, np.float32, "positive", s)
    assert p.min() >= 0.0 and p.max() < 1.0
    i = synth.vector(1 << 16, np.int32, "uniform", s)
    assert i.min() == -128 and i.max() == 127
    si = synth.vector(1 << 12, np.float32, "smallint", s)
    assert set(np.unique(si).tolist()) == {-1.0, 0.0, 1.0}
    s4 = synth.vector(1 << 12, np.int32, "smallint4", s)
    assert s4.min() == -4 and s4.max() == 4


def test_scalar_value_formula():
    s = 99
    h = synth.hash_scalar(s, 5)
    expect = ((((h >> 40) & 0xFFFFFF) - 2**23) * 2.0**-23)
    assert synth.vector(6, np.float32, "uniform", s)[5] == np.float32(expect)
    expect_i = ((h >> 56) & 0xFF) - 128
    assert synth.vector(6, np.int32, "uniform", s)[5] == expect_i


def test_layouts_and_blocks_are_slices_of_one_logical_matrix():
    R, C, s = 13, 29, 7
    A = synth.matrix(R, C, "mv", np.float32, "uniform", s)
    B = synth.matrix(R, C, "tmv", np.float32, "uniform", s)
    assert np.array_equal(B, A.T)
    blk = synth.matrix(R, C, "mv", np.float32, "uniform", s, rows=(3, 9), cols=(4, 20))
    assert np.array_equal(blk, A[3:9, 4:20])
    blkt = synth.matrix(R, C, "tmv", np.float32, "uniform", s, rows=(3, 9), cols=(4, 20))
    assert np.array_equal(blkt, A[3:9, 4:20].T)
    x = synth.vector(C, np.float32, "uniform", s)
    assert np.array_equal(synth.vector(10, np.float32, "uniform", s, start=5), x[5:15])
    # a(r, c) is hashed at logical index r*C + c
    assert A[2, 3] == synth.vector(R * C, np.float32, "uniform", s)[2 * C + 3]


def test_rowscale():
    R, C = 50, 8
    A = synth.matrix(R, C, "mv", np.float32, "uniform", 3)
    S = synth.matrix(R, C, "mv", np.float32, "rowscale", 3)
    for r in range(R):
        assert np.array_equal(S[r], A[r] * np.float32(2.0 ** ((r % 41) - 20)))
