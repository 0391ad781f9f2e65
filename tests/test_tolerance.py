"""P14: the fp32 tolerance |y - y_ref| <= 1e-4 * S_r (north_star) is provable for
the kernels' summation structure, and fails without the chain-length rule.

Standard bound (Higham, Accuracy and Stability of Numerical Algorithms, eq. 4.4):
a sum evaluated by any tree whose longest root-to-leaf path has m additions
(plus one rounding for each FMA product) satisfies |err| <= gamma_m * sum|p_i|,
gamma_m = m*u / (1 - m*u), u = 2^-24.  The kernels cap each thread's serial
chain at 1024 terms, followed by <= 40 tree levels.
"""
import numpy as np

U32 = 2.0 ** -24


def gamma(m):
    return m * U32 / (1 - m * U32)


def test_bound_with_chain_cap_is_below_tolerance():
    m = 1024 + 40 + 1           # chain + tree depth over all partials + product rounding
    assert gamma(m) < 1e-4
    assert gamma(1677) <= 1e-4 < gamma(1679)  # the largest admissible m


def test_serial_chain_on_positive_data_breaks_tolerance():
    """Why the cap exists: a single fp32 running sum over 2^20 equal positive
    terms (0.1f) is off by ~1e-2 relative -- 100x the tolerance -- because every
    addition rounds the same way once the sum is large."""
    n = 1 << 20
    p = np.full(n, 0.1, dtype=np.float32)
    serial = np.cumsum(p, dtype=np.float32)[-1]         # strictly sequential fp32 sum
    exact = p.astype(np.float64).sum()
    assert abs(float(serial) - exact) > 1e-4 * exact
    # the chunked scheme the kernels use (chain <= 1024, then a pairwise tree) passes
    parts = p.reshape(-1, 1024)
    chunk = np.cumsum(parts, axis=1, dtype=np.float32)[:, -1]
    while chunk.size > 1:
        chunk = (chunk[0::2] + chunk[1::2]).astype(np.float32)
    assert abs(float(chunk[0]) - exact) <= gamma(1024 + 12 + 1) * exact
