"""CPU oracle for the Adaptic hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
``paper_conf_pldi_samadihmlm12_b200`` never imports it, and the C source
(``oracle/oracle.c``) shares nothing with the CUDA path.

Every function is a thin ctypes marshaller around ``oracle.c``; the arithmetic
and its paper citations live there:

* :func:`mv`  -- y_r = sum_c A[r, c] x[c]
* :func:`tmv` -- y_r = sum_c B[c, r] x[c], B = A^T  (Fig. 3)
* :func:`dot` -- y_n = sum_e a[n, e] b[n, e]
* :func:`rows` -- selected outputs of MV/TMV, one by one (full-size configs)
* :func:`restructure` -- the Fig. 3 address map

float32 inputs return ``(y, S)`` in float64 with ``S_r = sum |a x|`` (tolerance
``|y_gpu - y| <= 1e-4 S``); int32 inputs return int32 computed modulo 2^32.

Pins: ``tests/test_oracle.py`` (P1-P14 of SURVEY.md section 8(c)).  No function
here is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared", "-std=c11"]


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (plain C, no OpenMP, no fast-math)."""
    if force or not os.path.exists(_LIB_PATH) or \
            os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        tmp = _LIB_PATH + ".tmp.%d" % os.getpid()
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        P = ctypes.c_void_p
        I = ctypes.c_int64
        for name in ("oracle_mv_f64", "oracle_tmv_f64", "oracle_dot_f64"):
            f = getattr(lib, name)
            f.argtypes = [P, P, I, I, P, P]
            f.restype = ctypes.c_int
        for name in ("oracle_mv_u32", "oracle_tmv_u32", "oracle_dot_u32"):
            f = getattr(lib, name)
            f.argtypes = [P, P, I, I, P]
            f.restype = ctypes.c_int
        lib.oracle_rows_f64.argtypes = [ctypes.c_int, P, P, I, I, P, I, P, P]
        lib.oracle_rows_f64.restype = ctypes.c_int
        lib.oracle_rows_u32.argtypes = [ctypes.c_int, P, P, I, I, P, I, P]
        lib.oracle_rows_u32.restype = ctypes.c_int
        lib.oracle_restructure_f32.argtypes = [P, I, I, P]
        lib.oracle_restructure_f32.restype = ctypes.c_int
        _lib = lib
    return _lib


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


def _c(a, dtype):
    a = np.ascontiguousarray(a)
    if a.dtype != dtype:
        raise TypeError(f"oracle expects {np.dtype(dtype)}, got {a.dtype}")
    return a


def _run(kind: str, M, x, R: int, C: int):
    lib = _load()
    R, C = int(R), int(C)
    if M.dtype == np.float32:
        M = _c(M, np.float32)
        x = _c(x, np.float32)
        y = np.empty(R, np.float64)
        S = np.empty(R, np.float64)
        rc = getattr(lib, f"oracle_{kind}_f64")(_ptr(M), _ptr(x), R, C, _ptr(y), _ptr(S))
        if rc:
            raise ValueError(f"oracle_{kind}_f64 rc={rc}")
        return y, S
    if M.dtype == np.int32:
        M = _c(M, np.int32)
        x = _c(x, np.int32)
        y = np.empty(R, np.int32)
        rc = getattr(lib, f"oracle_{kind}_u32")(_ptr(M), _ptr(x), R, C, _ptr(y))
        if rc:
            raise ValueError(f"oracle_{kind}_u32 rc={rc}")
        return y
    raise TypeError(f"unsupported dtype {M.dtype}")


def mv(A: np.ndarray, x: np.ndarray):
    """MV: A is R x C row-major (contiguous reductions)."""
    R, C = A.shape
    assert x.shape == (C,)
    return _run("mv", A, x, R, C)


def tmv(B: np.ndarray, x: np.ndarray):
    """TMV: B is C x R row-major (B = A^T); returns R outputs."""
    C, R = B.shape
    assert x.shape == (C,)
    return _run("tmv", B, x, R, C)


def dot(a: np.ndarray, b: np.ndarray):
    """Scalar products of N pairs: a, b are N x L row-major."""
    N, L = a.shape
    assert b.shape == (N, L)
    return _run("dot", a, b, N, L)


def rows(layout: str, M: np.ndarray, x: np.ndarray, R: int, C: int, idx):
    """Outputs ``idx`` of MV (layout 'mv', M is R x C) or TMV ('tmv', M is C x R)."""
    lib = _load()
    idx = np.ascontiguousarray(np.asarray(idx, dtype=np.int64))
    lay = {"mv": 0, "tmv": 1}[layout]
    if M.dtype == np.float32:
        M = _c(M, np.float32)
        x = _c(x, np.float32)
        y = np.empty(len(idx), np.float64)
        S = np.empty(len(idx), np.float64)
        rc = lib.oracle_rows_f64(lay, _ptr(M), _ptr(x), int(R), int(C), _ptr(idx), len(idx),
                                 _ptr(y), _ptr(S))
        if rc:
            raise ValueError(f"oracle_rows_f64 rc={rc}")
        return y, S
    M = _c(M, np.int32)
    x = _c(x, np.int32)
    y = np.empty(len(idx), np.int32)
    rc = lib.oracle_rows_u32(lay, _ptr(M), _ptr(x), int(R), int(C), _ptr(idx), len(idx), _ptr(y))
    if rc:
        raise ValueError(f"oracle_rows_u32 rc={rc}")
    return y


def restructure(buf: np.ndarray, T: int, P: int) -> np.ndarray:
    """Fig. 3 memory restructuring: out[T*k + t] = in[P*t + k]."""
    lib = _load()
    buf = _c(buf, np.float32)
    assert buf.size == T * P
    out = np.empty(T * P, np.float32)
    rc = lib.oracle_restructure_f32(_ptr(buf), int(T), int(P), _ptr(out))
    if rc:
        raise ValueError("oracle_restructure_f32 failed")
    return out


# ---------------------------------------------------------------- BLAS-1
def _blas1_lib():
    lib = _load()
    if not getattr(lib, "_blas1_ready", False):
        P, I = ctypes.c_void_p, ctypes.c_int64
        lib.oracle_asum_f64.argtypes = [P, I, I, P]
        lib.oracle_asum_f64.restype = ctypes.c_int
        lib.oracle_nrm2_f64.argtypes = [P, I, I, P, P]
        lib.oracle_nrm2_f64.restype = ctypes.c_int
        lib.oracle_iamaxmin.argtypes = [P, I, I, ctypes.c_int, P]
        lib.oracle_iamaxmin.restype = ctypes.c_int
        lib._blas1_ready = True
    return lib


def _rows2d(a):
    a = _c(a, np.float32)
    return a.reshape(1, -1) if a.ndim == 1 else a


def asum(a: np.ndarray) -> np.ndarray:
    """y_n = sum_e |a[n, e]| (float64)."""
    a = _rows2d(a)
    y = np.empty(a.shape[0], np.float64)
    assert _blas1_lib().oracle_asum_f64(_ptr(a), a.shape[0], a.shape[1], _ptr(y)) == 0
    return y


def nrm2(a: np.ndarray):
    """(y, ssq): y_n = sqrt(sum_e a[n, e]^2), ssq_n the sum of squares (float64)."""
    a = _rows2d(a)
    y = np.empty(a.shape[0], np.float64)
    s = np.empty(a.shape[0], np.float64)
    assert _blas1_lib().oracle_nrm2_f64(_ptr(a), a.shape[0], a.shape[1], _ptr(y), _ptr(s)) == 0
    return y, s


def iamax(a: np.ndarray) -> np.ndarray:
    """1-based first index of max |a[n, :]| (0 for empty rows), int64."""
    a = _rows2d(a)
    y = np.empty(a.shape[0], np.int64)
    assert _blas1_lib().oracle_iamaxmin(_ptr(a), a.shape[0], a.shape[1], 1, _ptr(y)) == 0
    return y


def iamin(a: np.ndarray) -> np.ndarray:
    """1-based first index of min |a[n, :]| (0 for empty rows), int64."""
    a = _rows2d(a)
    y = np.empty(a.shape[0], np.int64)
    assert _blas1_lib().oracle_iamaxmin(_ptr(a), a.shape[0], a.shape[1], -1, _ptr(y)) == 0
    return y


def stencil5(u: np.ndarray, c: float, n: float):
    """Five-point stencil of an H x W fp32 grid (oracle.c oracle_stencil5_f64): returns
    (v, S) in float64, v = c u + n (T + B + L + R) inside, v = u on the edge."""
    u = _c(u, np.float32)
    H, W = u.shape
    v = np.empty((H, W), np.float64)
    S = np.empty((H, W), np.float64)
    lib = _load()
    if not getattr(lib, "_st5_ready", False):
        P = ctypes.c_void_p
        I = ctypes.c_int64
        lib.oracle_stencil5_f64.argtypes = [P, I, I, ctypes.c_double, ctypes.c_double, P, P]
        lib.oracle_stencil5_f64.restype = ctypes.c_int
        lib._st5_ready = True
    assert lib.oracle_stencil5_f64(_ptr(u), H, W, float(c), float(n), _ptr(v), _ptr(S)) == 0
    return v, S
