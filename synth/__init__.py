"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the method (no products, no sums over a
row): it only turns (seed, logical index) into input values, so both the oracle
(``oracle/``) and the product path can be fed the same arrays.  A CUDA version
of the same counter-based generator lives in ``synth/synth_gen.cu`` (built to
``synth/libsynth.so``) for inputs too large to build on the host; the two are
cross-checked element by element in ``tests/test_synth.py`` (CPU: against a
pure-Python scalar splitmix64) and ``tests/test_gpu_parity.py`` (GPU).

Recipe (the paper states no
value distribution):

* logical element a(r, c) of an R x C problem has index i = r*C + c, whatever
  the physical layout (MV stores A[r, c], TMV stores B[c, r] = a(r, c)); a
  vector element x[c] has index i = c; so shards are slices of one logical array.
* h = splitmix64(seed XOR (i * 0x9E3779B97F4A7C15)), all arithmetic mod 2^64.
* kinds (fp32 / int32):
    uniform   : ((h>>40) & 0xFFFFFF) - 2^23) * 2^-23  in [-1, 1), exact in fp32
                ((h>>56) & 0xFF) - 128                 in [-128, 127]
    positive  : ((h>>40) & 0xFFFFFF) * 2^-24           in [0, 1)
                (h>>56) & 0x7F                         in [0, 127]
    ones      : 1
    smallint  : ((h>>40) mod 3) - 1                    in {-1, 0, 1}
    smallint4 : ((h>>40) mod 9) - 4                    in [-4, 4]
    identity  : 1 if r == c else 0          (matrices only)
    perm      : 1 if c == R-1-r else 0      (matrices only; the reversal permutation)
    diag      : uniform(i) if r == c else 0 (matrices only)
    rowscale  : uniform(i) * 2^((r mod 41) - 20)       (fp32 matrices only)
    diagdom   : uniform(i) if r != c else C            (matrices only; strictly diagonally
                dominant since |uniform| < 1: the BiCGSTAB systems)
* seeds: seed(config, role) = 20120611 + 1000*config + {A: 0, x: 1, b: 2}.
"""
from __future__ import annotations

import numpy as np

SEED_BASE = 20120611
GOLDEN_GAMMA = 0x9E3779B97F4A7C15
_M1 = 0xBF58476D1CE4E5B9
_M2 = 0x94D049BB133111EB
_MASK64 = (1 << 64) - 1

KINDS = ("uniform", "positive", "ones", "smallint", "smallint4",
         "identity", "perm", "diag", "rowscale", "diagdom")
VECTOR_KINDS = ("uniform", "positive", "ones", "smallint", "smallint4")
KIND_CODE = {k: i for i, k in enumerate(KINDS)}

_CHUNK = 1 << 22


def seed(config: int, role: str) -> int:
    return SEED_BASE + 1000 * int(config) + {"A": 0, "x": 1, "b": 2}[role]


def splitmix64_scalar(z: int) -> int:
    """Reference scalar splitmix64 finaliser (Steele, Lea, Flood 2014), pure Python."""
    z = (z + GOLDEN_GAMMA) & _MASK64
    z = ((z ^ (z >> 30)) * _M1) & _MASK64
    z = ((z ^ (z >> 27)) * _M2) & _MASK64
    return z ^ (z >> 31)


def hash_scalar(s: int, i: int) -> int:
    return splitmix64_scalar((s ^ ((i * GOLDEN_GAMMA) & _MASK64)) & _MASK64)


def hash64(s: int, idx: np.ndarray) -> np.ndarray:
    """Vectorised h = splitmix64(s ^ (idx * GAMMA)); uint64 arithmetic wraps."""
    z = np.asarray(idx, dtype=np.uint64) * np.uint64(GOLDEN_GAMMA)
    z ^= np.uint64(s & _MASK64)
    z += np.uint64(GOLDEN_GAMMA)
    z = (z ^ (z >> np.uint64(30))) * np.uint64(_M1)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(_M2)
    return z ^ (z >> np.uint64(31))


def _from_hash(h: np.ndarray, dtype, kind: str) -> np.ndarray:
    dtype = np.dtype(dtype)
    if kind in ("uniform", "diag", "rowscale", "diagdom"):
        if dtype == np.float32:
            v = ((h >> np.uint64(40)) & np.uint64(0xFFFFFF)).astype(np.int64) - (1 << 23)
            return (v.astype(np.float32) * np.float32(2.0 ** -23)).astype(np.float32)
        return (((h >> np.uint64(56)) & np.uint64(0xFF)).astype(np.int64) - 128).astype(np.int32)
    if kind == "positive":
        if dtype == np.float32:
            v = ((h >> np.uint64(40)) & np.uint64(0xFFFFFF)).astype(np.int64)
            return (v.astype(np.float32) * np.float32(2.0 ** -24)).astype(np.float32)
        return ((h >> np.uint64(56)) & np.uint64(0x7F)).astype(np.int32)
    if kind == "smallint":
        return ((h >> np.uint64(40)) % np.uint64(3)).astype(np.int64).astype(dtype) - dtype.type(1)
    if kind == "smallint4":
        return ((h >> np.uint64(40)) % np.uint64(9)).astype(np.int64).astype(dtype) - dtype.type(4)
    raise ValueError(kind)


def vector(n: int, dtype, kind: str, s: int, start: int = 0) -> np.ndarray:
    """x[c] for c in [start, start+n)."""
    if kind not in VECTOR_KINDS:
        raise ValueError(f"{kind} is not a vector kind")
    dtype = np.dtype(dtype)
    if kind == "ones":
        return np.ones(n, dtype)
    out = np.empty(n, dtype)
    for a in range(0, n, _CHUNK):
        b = min(n, a + _CHUNK)
        idx = np.arange(start + a, start + b, dtype=np.uint64)
        out[a:b] = _from_hash(hash64(s, idx), dtype, kind)
    return out


def matrix(R: int, C: int, layout: str, dtype, kind: str, s: int,
           rows=None, cols=None) -> np.ndarray:
    """The logical R x C matrix a(r, c) (or its [r0,r1) x [c0,c1) block) stored in
    ``layout``: 'mv' -> array[r - r0, c - c0]; 'tmv' -> array[c - c0, r - r0]."""
    dtype = np.dtype(dtype)
    if kind not in KINDS:
        raise ValueError(kind)
    r0, r1 = rows if rows is not None else (0, R)
    c0, c1 = cols if cols is not None else (0, C)
    nr, nc = r1 - r0, c1 - c0
    a = np.empty((nr, nc), dtype)
    step = max(1, _CHUNK // max(1, nc))
    for ra in range(0, nr, step):
        rb = min(nr, ra + step)
        r = np.arange(r0 + ra, r0 + rb, dtype=np.int64)[:, None]
        c = np.arange(c0, c1, dtype=np.int64)[None, :]
        if kind == "ones":
            blk = np.ones((rb - ra, nc), dtype)
        elif kind == "identity":
            blk = (r == c).astype(dtype)
        elif kind == "perm":
            blk = (c == (R - 1 - r)).astype(dtype)
        else:
            idx = (r * C + c).astype(np.uint64)
            blk = _from_hash(hash64(s, idx), dtype, kind)
            if kind == "diag":
                blk = np.where(r == c, blk, dtype.type(0)).astype(dtype)
            elif kind == "diagdom":
                blk = np.where(r == c, dtype.type(C), blk).astype(dtype)
            elif kind == "rowscale":
                if dtype != np.float32:
                    raise ValueError("rowscale is fp32 only")
                scale = np.ldexp(np.float32(1.0), ((r % 41) - 20).astype(np.int32))
                blk = (blk * scale.astype(np.float32)).astype(np.float32)
        a[ra:rb] = blk
    if layout == "mv":
        return a
    if layout == "tmv":
        return np.ascontiguousarray(a.T)
    raise ValueError(layout)


# ---------------------------------------------------------------------------- device copy
_dev_lib = None


def _device_lib():
    """ctypes handle of synth/libsynth.so (the CUDA twin of this generator)."""
    global _dev_lib
    if _dev_lib is None:
        import ctypes
        import os
        path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libsynth.so")
        if not os.path.exists(path):
            build_device()
        L = ctypes.CDLL(path)
        vp, i32, i64, u64 = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64, ctypes.c_uint64
        L.synth_fill_matrix.argtypes = [vp, i32, i32, i32, u64, i64, i64, i64, i64, i64, i64, vp]
        L.synth_fill_matrix.restype = i32
        L.synth_fill_vector.argtypes = [vp, i32, i32, u64, i64, i64, vp]
        L.synth_fill_vector.restype = i32
        _dev_lib = L
    return _dev_lib


def build_device(force: bool = False) -> str:
    import os
    import subprocess
    here = os.path.dirname(os.path.abspath(__file__))
    src, out = os.path.join(here, "synth_gen.cu"), os.path.join(here, "libsynth.so")
    if force or not os.path.exists(out) or os.path.getmtime(out) < os.path.getmtime(src):
        tmp = out + ".tmp.%d" % os.getpid()
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a",
                               "-O3", "-std=c++17", "-Xcompiler", "-fPIC", "-shared", "-o", tmp, src])
        os.replace(tmp, out)
    return out


def device_matrix(t, R: int, C: int, layout: str, kind: str, s: int, rows=None, cols=None, stream: int = 0):
    """Fill the CUDA tensor ``t`` (float32/int32, contiguous) with the [r0,r1) x [c0,c1)
    block of the logical matrix, in ``layout`` -- same values as :func:`matrix`."""
    import torch
    r0, r1 = rows if rows is not None else (0, R)
    c0, c1 = cols if cols is not None else (0, C)
    assert t.is_cuda and t.is_contiguous() and t.numel() == (r1 - r0) * (c1 - c0)
    dt = {torch.float32: 0, torch.int32: 1}[t.dtype]
    rc = _device_lib().synth_fill_matrix(t.data_ptr(), dt, {"mv": 0, "tmv": 1}[layout], KIND_CODE[kind],
                                         s & _MASK64, R, C, r0, r1, c0, c1, stream or None)
    if rc:
        raise RuntimeError(f"synth_fill_matrix cuda error {rc}")
    return t


def device_vector(t, kind: str, s: int, start: int = 0, stream: int = 0):
    import torch
    assert t.is_cuda and t.is_contiguous()
    if kind not in VECTOR_KINDS:
        raise ValueError(kind)
    dt = {torch.float32: 0, torch.int32: 1}[t.dtype]
    rc = _device_lib().synth_fill_vector(t.data_ptr(), dt, KIND_CODE[kind], s & _MASK64, start, t.numel(),
                                         stream or None)
    if rc:
        raise RuntimeError(f"synth_fill_vector cuda error {rc}")
    return t
