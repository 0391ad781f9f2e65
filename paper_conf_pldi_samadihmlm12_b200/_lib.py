"""ctypes binding of ``libadaptic.so`` (the C ABI declared in ``include/adaptic.h``).

Argument marshalling only: every operation of the hot path runs in the CUDA
kernels behind these entry points.  There is no fallback -- if the library is
missing or fails to load, :func:`lib` raises.
"""
from __future__ import annotations

import ctypes
import json
import os
import threading

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("ADAPTIC_LIB", os.path.join(HERE, "libadaptic.so"))

# enums (mirror include/adaptic.h)
OK, ERR_INVALID_ARG, ERR_UNSUPPORTED, ERR_MISALIGNED, ERR_ALIAS, ERR_NO_WORKSPACE, ERR_CUDA = range(7)
OP_MV, OP_TMV, OP_DOT = 0, 1, 2
OP_ASUM, OP_NRM2, OP_IAMAX, OP_IAMIN, OP_B1ALL, OP_STENCIL5 = 3, 4, 5, 6, 7, 8
OPS = {"mv": OP_MV, "tmv": OP_TMV, "dot": OP_DOT, "asum": OP_ASUM, "nrm2": OP_NRM2,
       "iamax": OP_IAMAX, "iamin": OP_IAMIN, "b1all": OP_B1ALL, "stencil5": OP_STENCIL5}
B1_VARIANTS = ("MV_SUBWARP", "MV_WPR", "MV_CPR", "MV_SPLIT")
F32, I32 = 0, 1
VARIANTS = ("AUTO", "MV_TPR", "MV_SUBWARP", "MV_WPR", "MV_CPR", "MV_SPLIT",
            "TMV_COL", "TMV_SPLITK", "TMV_REGTILE", "ST_DIRECT", "ST_TILE")
ST_VARIANTS = ("ST_DIRECT", "ST_TILE")
V = {name: i for i, name in enumerate(VARIANTS)}
MV_VARIANTS = ("MV_TPR", "MV_SUBWARP", "MV_WPR", "MV_CPR", "MV_SPLIT")
TMV_VARIANTS = ("TMV_COL", "TMV_SPLITK", "TMV_REGTILE")
P_LANES, P_SPLITS, P_CTAS_PER_SM, P_UNROLL, P_XSMEM, P_BLOCK, P_ROWS, P_ORDER, P_PIPE, NPARAMS = 0, 1, 2, 3, 4, 5, 6, 7, 8, 9

# every symbol the header declares (tests check they are all exported)
SYMBOLS = ("adaptic_plan", "adaptic_plan_forced", "adaptic_plan_multi", "adaptic_plan_variant", "adaptic_plan_describe",
           "adaptic_plan_workspace_bytes", "adaptic_plan_set_workspace", "adaptic_run", "adaptic_run_batch",
           "adaptic_run_host", "adaptic_plan_destroy", "adaptic_status_string",
           "adaptic_variant_name", "adaptic_last_cuda_error", "adaptic_abi_version",
           "adaptic_bicgstab_create", "adaptic_bicgstab_workspace_bytes", "adaptic_bicgstab_set_workspace",
           "adaptic_bicgstab_start", "adaptic_bicgstab_iterate", "adaptic_bicgstab_state",
           "adaptic_bicgstab_solve", "adaptic_bicgstab_destroy")

_lib = None
_lock = threading.Lock()


class AdapticError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = lib().adaptic_status_string(status).decode()
        if status == ERR_CUDA:
            msg += f" (cudaError {lib().adaptic_last_cuda_error()})"
        super().__init__(f"{where}: {msg}")


def lib():
    """Load libadaptic.so (raises if it was not built -- there is no CPU fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    with _lock:
        if _lib is not None:
            return _lib
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(
                f"{LIB_PATH} not found: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
                "(or python -m paper_conf_pldi_samadihmlm12_b200.build_ext); there is no CPU fallback")
        L = ctypes.CDLL(LIB_PATH)
        vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
        L.adaptic_plan.argtypes = [i32, i64, i64, i32, ctypes.POINTER(vp)]
        L.adaptic_plan.restype = i32
        L.adaptic_plan_forced.argtypes = [i32, i64, i64, i32, i32, ctypes.POINTER(ctypes.c_int32),
                                          ctypes.POINTER(vp)]
        L.adaptic_plan_forced.restype = i32
        L.adaptic_plan_multi.argtypes = [i32, i64, i64, ctypes.c_int32, i32, i32, ctypes.POINTER(ctypes.c_int32),
                                         ctypes.POINTER(vp)]
        L.adaptic_plan_multi.restype = i32
        L.adaptic_plan_variant.argtypes = [vp]
        L.adaptic_plan_variant.restype = i32
        L.adaptic_plan_describe.argtypes = [vp, ctypes.c_char_p, ctypes.c_size_t]
        L.adaptic_plan_describe.restype = i32
        L.adaptic_plan_workspace_bytes.argtypes = [vp]
        L.adaptic_plan_workspace_bytes.restype = ctypes.c_size_t
        L.adaptic_plan_set_workspace.argtypes = [vp, vp, ctypes.c_size_t]
        L.adaptic_plan_set_workspace.restype = i32
        L.adaptic_run.argtypes = [vp, vp, vp, vp, vp]
        L.adaptic_run.restype = i32
        L.adaptic_run_batch.argtypes = [ctypes.c_int32, ctypes.POINTER(vp), ctypes.POINTER(vp), ctypes.POINTER(vp),
                                        ctypes.POINTER(vp), ctypes.c_int32, vp]
        L.adaptic_run_batch.restype = i32
        L.adaptic_run_host.argtypes = [vp, vp, vp, vp, vp, vp, vp, vp]
        L.adaptic_run_host.restype = i32
        L.adaptic_plan_destroy.argtypes = [vp]
        L.adaptic_plan_destroy.restype = None
        L.adaptic_status_string.argtypes = [i32]
        L.adaptic_status_string.restype = ctypes.c_char_p
        L.adaptic_variant_name.argtypes = [i32]
        L.adaptic_variant_name.restype = ctypes.c_char_p
        L.adaptic_last_cuda_error.argtypes = []
        L.adaptic_last_cuda_error.restype = i32
        L.adaptic_abi_version.argtypes = []
        L.adaptic_abi_version.restype = i32
        f32, pi32, pf32 = ctypes.c_float, ctypes.POINTER(ctypes.c_int32), ctypes.POINTER(ctypes.c_float)
        L.adaptic_bicgstab_create.argtypes = [i64, ctypes.POINTER(vp)]
        L.adaptic_bicgstab_create.restype = i32
        L.adaptic_bicgstab_workspace_bytes.argtypes = [vp]
        L.adaptic_bicgstab_workspace_bytes.restype = ctypes.c_size_t
        L.adaptic_bicgstab_set_workspace.argtypes = [vp, vp, ctypes.c_size_t]
        L.adaptic_bicgstab_set_workspace.restype = i32
        L.adaptic_bicgstab_start.argtypes = [vp, vp, vp, vp]
        L.adaptic_bicgstab_start.restype = i32
        L.adaptic_bicgstab_iterate.argtypes = [vp, vp, vp, ctypes.c_int32, f32, vp]
        L.adaptic_bicgstab_iterate.restype = i32
        L.adaptic_bicgstab_state.argtypes = [vp, pi32, pf32, pi32, vp]
        L.adaptic_bicgstab_state.restype = i32
        L.adaptic_bicgstab_solve.argtypes = [vp, vp, vp, vp, ctypes.c_int32, f32, ctypes.c_int32, pi32, pf32, vp]
        L.adaptic_bicgstab_solve.restype = i32
        L.adaptic_bicgstab_destroy.argtypes = [vp]
        L.adaptic_bicgstab_destroy.restype = None
        _lib = L
    return _lib


def _check(status: int, where: str):
    if status != OK:
        raise AdapticError(status, where)


class Batch:
    """Marshalled arguments of adaptic_run_batch for a fixed list of (plan, A, x, y)."""

    def __init__(self, items):
        n = len(items)
        self.n = n
        self._plans = [it[0] for it in items]                 # keep the plans alive
        arr = lambda vals: (ctypes.c_void_p * max(1, n))(*[ctypes.c_void_p(v or None) for v in vals])  # noqa: E731
        self.plans = (ctypes.c_void_p * max(1, n))(*[p.handle for p in self._plans])
        self.A = arr([it[1] for it in items])
        self.x = arr([it[2] for it in items])
        self.y = arr([it[3] for it in items])

    def run(self, streams: int, stream: int = 0):
        _check(lib().adaptic_run_batch(self.n, self.plans, self.A, self.x, self.y, int(streams),
                                       ctypes.c_void_p(stream or None)), "adaptic_run_batch")


class Plan:
    """An ``adaptic_plan_t`` (selector output).  ``variant='AUTO'`` runs the selector."""

    def __init__(self, op: int, rows: int, cols: int, dtype: int, variant="AUTO", params=None, nvec: int = 1):
        L = lib()
        h = ctypes.c_void_p()
        v = V[variant] if isinstance(variant, str) else int(variant)
        if nvec != 1:
            arr = None
            if params is not None:
                vals = list(params) + [0] * (NPARAMS - len(params))
                arr = (ctypes.c_int32 * NPARAMS)(*vals)
            st = L.adaptic_plan_multi(op, int(rows), int(cols), int(nvec), dtype, v, arr, ctypes.byref(h))
        elif v == 0 and params is None:
            st = L.adaptic_plan(op, int(rows), int(cols), dtype, ctypes.byref(h))
        else:
            arr = None
            if params is not None:
                vals = list(params) + [0] * (NPARAMS - len(params))
                arr = (ctypes.c_int32 * NPARAMS)(*vals)
            st = L.adaptic_plan_forced(op, int(rows), int(cols), dtype, v, arr, ctypes.byref(h))
        _check(st, f"adaptic_plan({op},{rows},{cols},{dtype},{variant})")
        self._h = h
        self.op, self.rows, self.cols, self.dtype, self.nvec = op, int(rows), int(cols), dtype, int(nvec)

    @property
    def handle(self):
        return self._h

    @property
    def variant(self) -> str:
        return VARIANTS[lib().adaptic_plan_variant(self._h)]

    @property
    def workspace_bytes(self) -> int:
        return int(lib().adaptic_plan_workspace_bytes(self._h))

    def describe(self) -> dict:
        buf = ctypes.create_string_buffer(2048)
        n = lib().adaptic_plan_describe(self._h, buf, 2048)
        if n < 0:
            raise RuntimeError("adaptic_plan_describe failed")
        return json.loads(buf.value.decode())

    def set_workspace(self, ptr: int, nbytes: int):
        _check(lib().adaptic_plan_set_workspace(self._h, ctypes.c_void_p(ptr or None), nbytes),
               "adaptic_plan_set_workspace")

    def run_ptrs(self, A: int, x: int, y: int, stream: int = 0) -> int:
        """Raw entry: device pointers and a cudaStream_t as ints.  Returns the status."""
        return lib().adaptic_run(self._h, ctypes.c_void_p(A or None), ctypes.c_void_p(x or None),
                                 ctypes.c_void_p(y or None), ctypes.c_void_p(stream or None))

    def run(self, A: int, x: int, y: int, stream: int = 0):
        _check(self.run_ptrs(A, x, y, stream), "adaptic_run")

    def run_host(self, A_h: int, x_h: int, y_h: int, dA: int, dx: int, dy: int, stream: int = 0):
        _check(lib().adaptic_run_host(self._h, *(ctypes.c_void_p(p or None) for p in
                                                 (A_h, x_h, y_h, dA, dx, dy, stream))),
               "adaptic_run_host")

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value and _lib is not None:
            _lib.adaptic_plan_destroy(h)
            self._h = None


class BiCGSTAB:
    """An ``adaptic_bicgstab_t`` (BiCGSTAB on the adaptive MV; include/adaptic.h)."""

    def __init__(self, n: int):
        h = ctypes.c_void_p()
        _check(lib().adaptic_bicgstab_create(int(n), ctypes.byref(h)), f"adaptic_bicgstab_create({n})")
        self._h = h
        self.n = int(n)

    @property
    def workspace_bytes(self) -> int:
        return int(lib().adaptic_bicgstab_workspace_bytes(self._h))

    def set_workspace(self, ptr: int, nbytes: int):
        _check(lib().adaptic_bicgstab_set_workspace(self._h, ctypes.c_void_p(ptr or None), nbytes),
               "adaptic_bicgstab_set_workspace")

    def start(self, b: int, x: int, stream: int = 0):
        _check(lib().adaptic_bicgstab_start(self._h, ctypes.c_void_p(b or None), ctypes.c_void_p(x or None),
                                            ctypes.c_void_p(stream or None)), "adaptic_bicgstab_start")

    def iterate(self, A: int, x: int, iters: int, tol: float, stream: int = 0):
        _check(lib().adaptic_bicgstab_iterate(self._h, ctypes.c_void_p(A or None), ctypes.c_void_p(x or None),
                                              int(iters), float(tol), ctypes.c_void_p(stream or None)),
               "adaptic_bicgstab_iterate")

    def state(self, stream: int = 0):
        it, rel, done = ctypes.c_int32(), ctypes.c_float(), ctypes.c_int32()
        _check(lib().adaptic_bicgstab_state(self._h, ctypes.byref(it), ctypes.byref(rel), ctypes.byref(done),
                                            ctypes.c_void_p(stream or None)), "adaptic_bicgstab_state")
        return it.value, rel.value, done.value

    def solve(self, A: int, b: int, x: int, max_iters: int, tol: float, check_every: int = 8, stream: int = 0):
        it, rel = ctypes.c_int32(), ctypes.c_float()
        _check(lib().adaptic_bicgstab_solve(self._h, *(ctypes.c_void_p(p or None) for p in (A, b, x)),
                                            int(max_iters), float(tol), int(check_every), ctypes.byref(it),
                                            ctypes.byref(rel), ctypes.c_void_p(stream or None)),
               "adaptic_bicgstab_solve")
        return it.value, rel.value

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value and _lib is not None:
            _lib.adaptic_bicgstab_destroy(h)
            self._h = None
