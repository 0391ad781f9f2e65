"""PyTorch-facing API: ``mv``, ``tmv``, ``dot`` and the BLAS-1 reductions
``asum``, ``nrm2``, ``iamax``, ``iamin`` on CUDA tensors.

PyTorch supplies device memory and the stream; the selector
(``adaptic_plan``) and the kernels (``adaptic_run``) are the C ABI.  This module
only checks shapes/dtypes, allocates ``y`` and the zero-filled workspace the
split variants need, and caches plans per (op, shape, dtype, variant, device,
stream) so repeated calls cost one ctypes call.

Shapes (``include/adaptic.h``; reading R1):
  mv(A[R, C], x[C])      -> y[R],  y_r = sum_c A[r, c] x[c]
  tmv(B[C, R], x[C])     -> y[R],  y_r = sum_c B[c, r] x[c]   (B = A^T)
  dot(a[N, L], b[N, L])  -> y[N],  y_n = sum_e a[n, e] b[n, e]  (1-D a, b: N = 1)
dtype float32 (fp32 accumulate) or int32 (modulo 2^32).
"""
from __future__ import annotations

import threading

import torch

from . import _lib as L

_DT = {torch.float32: L.F32, torch.int32: L.I32}
_cache: dict = {}
_cache_lock = threading.Lock()


def _dtype_code(t: torch.Tensor) -> int:
    try:
        return _DT[t.dtype]
    except KeyError:
        raise TypeError(f"adaptic supports float32 and int32, got {t.dtype}") from None


def get_plan(op: int, rows: int, cols: int, dtype: int, device: torch.device,
             variant="AUTO", params=None, stream: int = 0, nvec: int = 1) -> L.Plan:
    """Cached plan with its workspace attached (allocated zero-filled on `device`)."""
    key = (op, int(rows), int(cols), dtype, variant, tuple(params) if params else None,
           device.index, stream, int(nvec))
    with _cache_lock:
        ent = _cache.get(key)
        if ent is not None:
            return ent[0]
    plan = L.Plan(op, rows, cols, dtype, variant, params, nvec)
    ws = None
    nbytes = plan.workspace_bytes
    if nbytes:
        ws = torch.zeros(nbytes, dtype=torch.uint8, device=device)
        plan.set_workspace(ws.data_ptr(), nbytes)
    with _cache_lock:
        _cache.setdefault(key, (plan, ws))
        return _cache[key][0]


def clear_cache():
    with _cache_lock:
        _cache.clear()


def _check_dev(*ts: torch.Tensor):
    dev = ts[0].device
    for t in ts:
        if t.device.type != "cuda":
            raise ValueError("adaptic runs on CUDA tensors only (there is no CPU path)")
        if t.device != dev:
            raise ValueError("all tensors must be on the same device")
        if not t.is_contiguous():
            raise ValueError("tensors must be contiguous (row-major)")
        if t.dtype != ts[0].dtype:
            raise TypeError("A and x must have the same dtype")
    return dev


def _run(op: int, M: torch.Tensor, X: torch.Tensor, R: int, C: int, variant, params, out):
    dev = _check_dev(M, X)
    dt = _dtype_code(M)
    if out is None:
        out = torch.empty(R, dtype=M.dtype, device=dev)
    else:
        _check_dev(M, out)
        if out.numel() != R:
            raise ValueError(f"out must have {R} elements")
    stream = torch.cuda.current_stream(dev).cuda_stream
    plan = get_plan(op, R, C, dt, dev, variant, params, stream)
    plan.run(M.data_ptr(), X.data_ptr(), out.data_ptr(), stream)
    return out


def mv(A: torch.Tensor, x: torch.Tensor, *, variant="AUTO", params=None, out=None) -> torch.Tensor:
    """y = A x for a row-major R x C matrix A (contiguous reductions)."""
    if A.dim() != 2 or x.dim() != 1 or x.shape[0] != A.shape[1]:
        raise ValueError(f"mv: A must be [R, C] and x [C], got {tuple(A.shape)}, {tuple(x.shape)}")
    return _run(L.OP_MV, A, x, A.shape[0], A.shape[1], variant, params, out)


def tmv(B: torch.Tensor, x: torch.Tensor, *, variant="AUTO", params=None, out=None) -> torch.Tensor:
    """y = B^T x for a row-major C x R matrix B (the restructured layout; y has R entries)."""
    if B.dim() != 2 or x.dim() != 1 or x.shape[0] != B.shape[0]:
        raise ValueError(f"tmv: B must be [C, R] and x [C], got {tuple(B.shape)}, {tuple(x.shape)}")
    return _run(L.OP_TMV, B, x, B.shape[1], B.shape[0], variant, params, out)


def dot(a: torch.Tensor, b: torch.Tensor, *, variant="AUTO", params=None, out=None) -> torch.Tensor:
    """Scalar products of N pairs: y[n] = <a[n], b[n]>; 1-D inputs are one pair."""
    if a.shape != b.shape or a.dim() not in (1, 2):
        raise ValueError(f"dot: a and b must both be [N, L] (or [L]), got {tuple(a.shape)}, {tuple(b.shape)}")
    N, Lk = (1, a.shape[0]) if a.dim() == 1 else a.shape
    return _run(L.OP_DOT, a, b, N, Lk, variant, params, out)


def _blas1(op: int, a: torch.Tensor, variant, params, out, ydtype) -> torch.Tensor:
    if a.dim() not in (1, 2):
        raise ValueError(f"expected [N, L] (or [L]) input, got {tuple(a.shape)}")
    if a.dtype != torch.float32:
        raise TypeError(f"BLAS-1 reductions take float32, got {a.dtype}")
    N, Lk = (1, a.shape[0]) if a.dim() == 1 else a.shape
    dev = _check_dev(a)
    if out is None:
        out = torch.empty(N, dtype=ydtype, device=dev)
    elif out.numel() != N or out.dtype != ydtype or out.device != dev or not out.is_contiguous():
        raise ValueError(f"out must be a contiguous {ydtype} tensor of {N} elements on {dev}")
    stream = torch.cuda.current_stream(dev).cuda_stream
    plan = get_plan(op, N, Lk, L.F32, dev, variant, params, stream)
    plan.run(a.data_ptr(), 0, out.data_ptr(), stream)
    return out


def asum(a: torch.Tensor, *, variant="AUTO", params=None, out=None) -> torch.Tensor:
    """Sasum per row: y[n] = sum_e |a[n, e]| (float32)."""
    return _blas1(L.OP_ASUM, a, variant, params, out, torch.float32)


def nrm2(a: torch.Tensor, *, variant="AUTO", params=None, out=None) -> torch.Tensor:
    """Snrm2 per row: y[n] = sqrt(sum_e a[n, e]^2) (float32; fp64 accumulation)."""
    return _blas1(L.OP_NRM2, a, variant, params, out, torch.float32)


def iamax(a: torch.Tensor, *, variant="AUTO", params=None, out=None) -> torch.Tensor:
    """Isamax per row: smallest 1-based index of max |a[n, e]| (int32; 0 for empty rows)."""
    return _blas1(L.OP_IAMAX, a, variant, params, out, torch.int32)


def iamin(a: torch.Tensor, *, variant="AUTO", params=None, out=None) -> torch.Tensor:
    """Isamin per row: smallest 1-based index of min |a[n, e]| (int32; 0 for empty rows)."""
    return _blas1(L.OP_IAMIN, a, variant, params, out, torch.int32)


MULTI_SIZES = (8, 4, 2, 1)


def _multi(op: int, M: torch.Tensor, X: torch.Tensor, R: int, C: int, variant, params, out):
    if X.dim() != 2 or X.shape[1] != C:
        raise ValueError(f"X must be [K, {C}], got {tuple(X.shape)}")
    dev = _check_dev(M, X)
    if M.dtype != torch.float32:
        raise TypeError("multi-vector forms take float32")
    K = X.shape[0]
    if out is None:
        out = torch.empty(K, R, dtype=M.dtype, device=dev)
    elif tuple(out.shape) != (K, R) or out.dtype != M.dtype or not out.is_contiguous():
        raise ValueError(f"out must be a contiguous float32 [{K}, {R}] tensor")
    stream = torch.cuda.current_stream(dev).cuda_stream
    j = 0
    while j < K:                       # the library runs K in {1, 2, 4, 8}: cover K greedily
        k = next(m for m in MULTI_SIZES if m <= K - j)
        plan = get_plan(op, R, C, L.F32, dev, variant if k > 1 else "AUTO", params if k > 1 else None, stream, k)
        plan.run(M.data_ptr(), X[j:j + k].data_ptr(), out[j:j + k].data_ptr(), stream)
        j += k
    return out


def mv_multi(A: torch.Tensor, X: torch.Tensor, *, variant="AUTO", params=None, out=None) -> torch.Tensor:
    """Y[j] = A X[j] for K vectors in one pass over A (horizontal actor integration,
    P:600).  A [R, C], X [K, C] -> Y [K, R], float32."""
    if A.dim() != 2:
        raise ValueError(f"mv_multi: A must be [R, C], got {tuple(A.shape)}")
    return _multi(L.OP_MV, A, X, A.shape[0], A.shape[1], variant, params, out)


def tmv_multi(B: torch.Tensor, X: torch.Tensor, *, variant="AUTO", params=None, out=None) -> torch.Tensor:
    """Y[j] = B^T X[j] for K vectors in one pass over B.  B [C, R], X [K, C] -> Y [K, R]."""
    if B.dim() != 2:
        raise ValueError(f"tmv_multi: B must be [C, R], got {tuple(B.shape)}")
    return _multi(L.OP_TMV, B, X, B.shape[1], B.shape[0], variant, params, out)


def b1all(a: torch.Tensor, *, variant="AUTO", params=None, out=None):
    """All four BLAS-1 reductions of every row from ONE pass over ``a`` (the paper's
    horizontal actor integration).  Returns (asum, nrm2, iamax, iamin): two
    float32 and two int32 tensors of N elements, views of one 16*N-byte buffer."""
    if a.dim() not in (1, 2):
        raise ValueError(f"expected [N, L] (or [L]) input, got {tuple(a.shape)}")
    if a.dtype != torch.float32:
        raise TypeError(f"BLAS-1 reductions take float32, got {a.dtype}")
    N, Lk = (1, a.shape[0]) if a.dim() == 1 else a.shape
    dev = _check_dev(a)
    if out is None:
        out = torch.empty(4 * N, dtype=torch.float32, device=dev)
    elif out.numel() != 4 * N or out.element_size() != 4 or out.device != dev or not out.is_contiguous():
        raise ValueError(f"out must be a contiguous 4-byte tensor of {4 * N} elements on {dev}")
    stream = torch.cuda.current_stream(dev).cuda_stream
    plan = get_plan(L.OP_B1ALL, N, Lk, L.F32, dev, variant, params, stream)
    plan.run(a.data_ptr(), 0, out.data_ptr(), stream)
    f = out.view(torch.float32)
    i = out.view(torch.int32)
    return f[:N], f[N:2 * N], i[2 * N:3 * N], i[3 * N:]


def plan(op: str, rows: int, cols: int, dtype: str = "f32", variant="AUTO", params=None, nvec: int = 1) -> L.Plan:
    """A bare plan (no workspace attached) -- for inspecting the selector."""
    return L.Plan(L.OPS[op], rows, cols, {"f32": L.F32, "i32": L.I32}[dtype], variant, params, nvec)


def run_host(op: str, M_host: torch.Tensor, X_host: torch.Tensor, y_host: torch.Tensor,
             dM: torch.Tensor, dX: torch.Tensor, dy: torch.Tensor, *, variant="AUTO"):
    """End-to-end call with HOST buffers (pinned for async copies): the library
    enqueues H2D copies of M and X into dM/dX, the kernel, and the D2H copy of y
    on the current stream.  The caller synchronises before reading y_host."""
    opc = L.OPS[op]
    if opc not in (L.OP_MV, L.OP_TMV, L.OP_DOT, L.OP_STENCIL5):
        raise ValueError(f"run_host supports mv, tmv, dot and stencil5, got {op!r}")
    if M_host.dim() not in (1, 2) or (opc != L.OP_DOT and M_host.dim() != 2):
        raise ValueError(f"run_host: bad matrix shape {tuple(M_host.shape)}")
    if opc == L.OP_TMV:
        C, R = M_host.shape
    elif M_host.dim() == 1:
        R, C = 1, M_host.shape[0]
    else:
        R, C = M_host.shape
    dev = _check_dev(dM, dX, dy)
    dt = _dtype_code(M_host)
    for t in (M_host, X_host, y_host):
        if t.device.type != "cpu" or not t.is_contiguous():
            raise ValueError("host buffers must be contiguous CPU tensors")
    # every buffer the library copies blindly must have the plan's size and dtype
    nx = R * C if opc == L.OP_DOT else 2 if opc == L.OP_STENCIL5 else C     # stencil: {c, n}
    ny = R * C if opc == L.OP_STENCIL5 else R
    want = {"M_host": (M_host, R * C), "X_host": (X_host, nx), "y_host": (y_host, ny),
            "dM": (dM, R * C), "dX": (dX, nx), "dy": (dy, ny)}
    for name, (t, n) in want.items():
        if t.dtype != M_host.dtype:
            raise TypeError(f"run_host: {name} is {t.dtype}, expected {M_host.dtype}")
        if t.numel() != n:
            raise ValueError(f"run_host: {name} has {t.numel()} elements, expected {n}")
    stream = torch.cuda.current_stream(dev).cuda_stream
    plan = get_plan(opc, R, C, dt, dev, variant, None, stream)
    plan.run_host(M_host.data_ptr(), X_host.data_ptr(), y_host.data_ptr(),
                  dM.data_ptr(), dX.data_ptr(), dy.data_ptr(), stream)
    return y_host


_solvers: dict = {}


def bicgstab_solver(n: int, device: torch.device, stream: int | None = None) -> "L.BiCGSTAB":
    """Cached solver for n x n systems on `device` with its zero-filled workspace.  The
    solver's vectors, MV workspace and device state are per solver, so the cache is keyed
    by the stream too (two streams never share one: their solves would race)."""
    if stream is None:
        stream = torch.cuda.current_stream(device).cuda_stream
    key = (int(n), device.index, int(stream or 0))
    with _cache_lock:
        ent = _solvers.get(key)
        if ent is not None:
            return ent[0]
    S = L.BiCGSTAB(n)
    ws = torch.zeros(S.workspace_bytes, dtype=torch.uint8, device=device)
    S.set_workspace(ws.data_ptr(), S.workspace_bytes)
    with _cache_lock:
        _solvers.setdefault(key, (S, ws))
        return _solvers[key][0]


def bicgstab(A: torch.Tensor, b: torch.Tensor, *, tol: float = 1e-6, max_iters: int = 1000,
             check_every: int = 8, out=None):
    """Solve A x = b (A [n, n] float32 CUDA, nonsymmetric) with BiCGSTAB on the adaptive MV
    (the paper's Sec. 5.2.2 case study).  Returns (x, iterations, relative residual)."""
    if A.dim() != 2 or A.shape[0] != A.shape[1] or b.shape != (A.shape[0],):
        raise ValueError(f"bicgstab: A must be [n, n] and b [n], got {tuple(A.shape)}, {tuple(b.shape)}")
    dev = _check_dev(A, b)
    if A.dtype != torch.float32:
        raise TypeError("bicgstab takes float32")
    if out is None:
        x = torch.empty_like(b)
    else:
        x = out
        if (x.dtype != torch.float32 or x.device != dev or not x.is_contiguous() or x.shape != b.shape):
            raise ValueError(f"out must be a contiguous float32 [{b.shape[0]}] tensor on {dev}")
        n4 = 4 * b.shape[0]
        for t, nb in ((b, n4), (A, n4 * A.shape[0])):
            if x.data_ptr() < t.data_ptr() + nb and t.data_ptr() < x.data_ptr() + n4:
                raise ValueError("out must not overlap A or b")
    stream = torch.cuda.current_stream(dev).cuda_stream
    S = bicgstab_solver(A.shape[0], dev, stream)
    it, rel = S.solve(A.data_ptr(), b.data_ptr(), x.data_ptr(), max_iters, tol, check_every, stream)
    return x, it, rel


_coefs: dict = {}


def stencil5(u: torch.Tensor, c: float, n: float, *, variant="AUTO", params=None, out=None) -> torch.Tensor:
    """Five-point stencil of an H x W float32 grid (the paper's neighbouring-access
    actor, Sec. 4.1.2): v = c u + n (T + B + L + R) inside, v = u on the edge."""
    if u.dim() != 2:
        raise ValueError(f"stencil5: u must be [H, W], got {tuple(u.shape)}")
    dev = _check_dev(u)
    if u.dtype != torch.float32:
        raise TypeError("stencil5 takes float32")
    H, W = u.shape
    key = (float(c), float(n), dev.index)
    coef = _coefs.get(key)
    if coef is None:
        coef = torch.tensor([c, n], dtype=torch.float32, device=dev)
        _coefs[key] = coef
    if out is None:
        out = torch.empty_like(u)
    elif out.shape != u.shape or out.dtype != u.dtype or not out.is_contiguous():
        raise ValueError("out must be a contiguous float32 tensor shaped like u")
    stream = torch.cuda.current_stream(dev).cuda_stream
    plan = get_plan(L.OP_STENCIL5, H, W, L.F32, dev, variant, params, stream)
    plan.run(u.data_ptr(), coef.data_ptr(), out.data_ptr(), stream)
    return out
