"""B200-native input-adaptive reductions (Adaptic, PLDI'12): MV, TMV, scalar product.

Public API (thin marshalling over the C ABI in ``include/adaptic.h``):

* :func:`mv`, :func:`tmv`, :func:`dot` -- run on CUDA tensors; the runtime
  selector picks the kernel variant from the actual (rows, cols).
* :func:`asum`, :func:`nrm2`, :func:`iamax`, :func:`iamin` -- BLAS-1 reductions
  (the paper's Fig. 9 CUBLAS benchmarks) on the same engine.
* :func:`plan` -- inspect what the selector picks (``Plan.describe()``).
* :mod:`.dist` -- multi-GPU row sharding and split-K over ``torch.distributed``.

There is no CPU fallback: without ``libadaptic.so`` every call raises.
"""
from ._lib import BiCGSTAB, VARIANTS, MV_VARIANTS, TMV_VARIANTS, AdapticError, Plan, lib  # noqa: F401
from .ops import (asum, b1all, bicgstab, bicgstab_solver, clear_cache, dot, get_plan, iamax, iamin, mv, mv_multi, nrm2, plan,  # noqa: F401
                  run_host, stencil5, tmv, tmv_multi)

__all__ = ["mv", "tmv", "dot", "asum", "nrm2", "iamax", "iamin", "b1all", "mv_multi", "tmv_multi", "bicgstab", "bicgstab_solver", "stencil5", "plan", "run_host", "Plan", "AdapticError", "lib",
           "VARIANTS", "MV_VARIANTS", "TMV_VARIANTS", "get_plan", "clear_cache"]
