"""Multi-GPU partitioning over ``torch.distributed`` (one process per GPU, NCCL).

Not in the paper (a single-GPU system); this is north_star item (4) and SURVEY.md
section 8(e).  The path shards naturally because every output is an independent
reduction ("each block computes the reduction output for one input array",
P:478):

* **Row shard** (MV, TMV, DOT with many outputs): rank g owns the contiguous
  output block ``shard_range(R, G, g)``; x is replicated; NO collective on the
  data path.  ``gather=True`` adds an all-gather of y (reported separately).
* **Split-K** (short-wide: few outputs, long reductions, BJ:configs[4]): rank g
  owns the contiguous reduction slice ``shard_range(C, G, g)`` (for TMV a
  contiguous block of B's rows), computes R partial sums with the local
  selected kernel, and the partials are combined across ranks -- the
  cross-GPU analogue of the paper's merge kernel:
    - fp32: ``all_reduce(SUM)`` (NCCL over NVLink/NVSwitch);
    - int32: ``all_gather`` of the G x R partials, then a fixed-order sum by the
      library's own TMV kernel with x = ones (y[r] = sum_g P[g, r] * 1, exact
      modulo 2^32), so the result is bit-exact by construction.

``partition`` is the rule that picks between the two (row blocks whenever every
rank gets at least ``ROW_MIN`` outputs, else split-K), and :class:`SplitKBucket`
combines the partials of MANY split-K problems with ONE collective per step
(the messages are R*4 bytes -- latency-bound -- so they are bucketed, not sent
one by one).

The local computations are the C-ABI kernels (``ops.mv/tmv/dot``); the
``local_fn`` / ``merge_fn`` hooks only let the host-side reassembly be exercised
on CPU with gloo (tests/test_dist.py).  tests/test_gpu_dist.py runs every entry
point WITHOUT them (gloo on CUDA tensors, world 2 and 3 on one GPU; NCCL world 1).
"""
from __future__ import annotations

from typing import Callable, Optional, Sequence

import torch
import torch.distributed as dist

from . import ops

ROW_MIN = 1024          # outputs per rank below which a problem is split along its reduction


def shard_range(n: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous block partition of [0, n): the first n % world ranks get one extra."""
    if world <= 0 or not 0 <= rank < world or n < 0:
        raise ValueError("bad shard arguments")
    base, rem = divmod(n, world)
    start = rank * base + min(rank, rem)
    return start, start + base + (1 if rank < rem else 0)


def partition(R: int, C: int, world: int, rank: int, row_min: int = ROW_MIN):
    """How rank ``rank`` of ``world`` shares the logical R x C reduction problem
    (R outputs, reduction length C -- reading R1).  Returns ``(kind, (r0, r1), (c0, c1))``:

    * ``"rows"``   -- outputs [r0, r1), the whole reduction; no collective;
    * ``"splitk"`` -- every output, reduction slice [c0, c1); partial sums must be
      combined across ranks (P:480's merge, over NVLink).

    Row blocks whenever every rank gets at least ``row_min`` outputs (or world == 1);
    split-K otherwise (north_star (4): "split-K ... where columns dominate")."""
    if world <= 0 or not 0 <= rank < world or R < 0 or C < 0:
        raise ValueError("bad partition arguments")
    if world == 1 or R >= world * row_min:
        return "rows", shard_range(R, world, rank), (0, C)
    return "splitk", (0, R), shard_range(C, world, rank)


def _world(group):
    return dist.get_world_size(group), dist.get_rank(group)


def mv_rowshard(A_local: torch.Tensor, x: torch.Tensor, *, group=None, gather: bool = False,
                local_fn: Optional[Callable] = None, variant="AUTO") -> torch.Tensor:
    """y rows of this rank's A block (R_local x C); optionally all-gathered to the full y.
    With gather=True every rank must hold shard_range-sized blocks."""
    fn = local_fn or (lambda A, xx: ops.mv(A, xx, variant=variant))
    y_local = fn(A_local, x)
    return gather_rows(y_local, group=group) if gather else y_local


def tmv_rowshard(B_local: torch.Tensor, x: torch.Tensor, *, group=None, gather: bool = False,
                 local_fn: Optional[Callable] = None, variant="AUTO") -> torch.Tensor:
    """TMV row shard: B_local is this rank's C x R_local block of B's columns (its own
    contiguous array); y_local = B_local^T x."""
    fn = local_fn or (lambda B, xx: ops.tmv(B, xx, variant=variant))
    y_local = fn(B_local, x)
    return gather_rows(y_local, group=group) if gather else y_local


def gather_rows(y_local: torch.Tensor, *, group=None) -> torch.Tensor:
    """All-gather variable-length row blocks (rank order) into the full y on every rank."""
    G, _ = _world(group)
    sizes = [None] * G
    dist.all_gather_object(sizes, int(y_local.numel()), group=group)
    width = max(sizes)                  # collectives need equal sizes: pad, gather, trim
    padded = torch.zeros(width, dtype=y_local.dtype, device=y_local.device)
    padded[: y_local.numel()] = y_local
    parts = torch.empty(G * width, dtype=y_local.dtype, device=y_local.device)
    dist.all_gather_into_tensor(parts, padded, group=group)
    return torch.cat([parts[g * width: g * width + s] for g, s in enumerate(sizes)])


def combine_splitk(y_part: torch.Tensor, *, group=None, merge_fn: Optional[Callable] = None,
                   inplace: bool = False) -> torch.Tensor:
    """Combine per-rank partial sums of the same R outputs into the full y (every rank).
    fp32: all_reduce(SUM); int32: all_gather + the library's fixed-order TMV merge."""
    if y_part.dtype == torch.float32:
        y = y_part if inplace else y_part.clone()
        dist.all_reduce(y, op=dist.ReduceOp.SUM, group=group)
        return y
    if y_part.dtype != torch.int32:
        raise TypeError("split-K combine supports float32 and int32")
    G, _ = _world(group)
    flat = y_part.contiguous().view(-1)
    P = torch.empty(G, flat.numel(), dtype=torch.int32, device=y_part.device)
    dist.all_gather_into_tensor(P.view(-1), flat, group=group)
    if merge_fn is not None:
        y = merge_fn(P)
        if inplace:
            y_part.view(-1).copy_(y)
            return y_part
        return y
    ones = torch.ones(G, dtype=torch.int32, device=P.device)
    if inplace:                         # y[r] = sum_g P[g, r] (mod 2^32), fixed order g = 0..G-1
        ops.tmv(P, ones, out=flat)
        return y_part
    return ops.tmv(P, ones)


class SplitKBucket:
    """One flat buffer holding the partial y of every split-K problem of a step, so the
    whole step needs ONE collective (all_reduce for fp32, all_gather + merge for int32)
    instead of one per problem.  ``views[i]`` is problem i's y (pass it as the kernel's
    output); after :meth:`combine` every view holds the full sums on every rank."""

    def __init__(self, sizes: Sequence[int], dtype: torch.dtype, device, group=None):
        if dtype not in (torch.float32, torch.int32):
            raise TypeError("split-K combine supports float32 and int32")
        self.sizes = [int(s) for s in sizes]
        self.group = group
        self.flat = torch.zeros(max(1, sum(self.sizes)), dtype=dtype, device=device)
        self.views, off = [], 0
        for s in self.sizes:
            self.views.append(self.flat[off: off + s])
            off += s
        self.nbytes = 4 * sum(self.sizes)
        if dtype == torch.int32 and self.sizes:
            G, _ = _world(group)
            self._P = torch.empty(G, self.flat.numel(), dtype=torch.int32, device=device)
            self._ones = torch.ones(G, dtype=torch.int32, device=device)

    def combine(self):
        if not self.sizes:
            return
        if self.flat.dtype == torch.float32:
            dist.all_reduce(self.flat, op=dist.ReduceOp.SUM, group=self.group)
        else:
            dist.all_gather_into_tensor(self._P.view(-1), self.flat, group=self.group)
            ops.tmv(self._P, self._ones, out=self.flat)


def tmv_splitk(B_local: torch.Tensor, x_local: torch.Tensor, *, group=None,
               local_fn: Optional[Callable] = None, merge_fn: Optional[Callable] = None,
               variant="AUTO") -> torch.Tensor:
    """B_local: this rank's contiguous rows [c0, c1) of the C x R matrix B; x_local = x[c0:c1].
    Returns the full y (R outputs) on every rank."""
    fn = local_fn or (lambda B, xx: ops.tmv(B, xx, variant=variant))
    return combine_splitk(fn(B_local, x_local), group=group, merge_fn=merge_fn, inplace=True)


def mv_splitk(A_local: torch.Tensor, x_local: torch.Tensor, *, group=None,
              local_fn: Optional[Callable] = None, merge_fn: Optional[Callable] = None,
              variant="AUTO") -> torch.Tensor:
    """A_local: this rank's column block of A, stored as its own R x C_local array."""
    fn = local_fn or (lambda A, xx: ops.mv(A, xx, variant=variant))
    return combine_splitk(fn(A_local, x_local), group=group, merge_fn=merge_fn, inplace=True)


def dot_splitk(a_local: torch.Tensor, b_local: torch.Tensor, *, group=None,
               local_fn: Optional[Callable] = None, merge_fn: Optional[Callable] = None,
               variant="AUTO") -> torch.Tensor:
    """Fewer pairs than ranks (e.g. Sdot, N = 1): split each pair's length."""
    fn = local_fn or (lambda a, b: ops.dot(a, b, variant=variant))
    return combine_splitk(fn(a_local, b_local), group=group, merge_fn=merge_fn, inplace=True)


def run_partitioned(op: str, M_local: torch.Tensor, X_local: torch.Tensor, R: int, C: int, *,
                    group=None, variant="AUTO", gather: bool = True) -> torch.Tensor:
    """One logical (op, R, C) problem, this rank's share held locally as ``partition``
    says: rows -> local kernel (+ all-gather of y if ``gather``); splitk -> local kernel
    + combine.  Returns the full y on every rank (or the local rows if not gather)."""
    G, g = _world(group)
    kind, (r0, r1), (c0, c1) = partition(R, C, G, g)
    fn = {"mv": ops.mv, "tmv": ops.tmv, "dot": ops.dot}[op]
    y = fn(M_local, X_local, variant=variant)
    if kind == "splitk":
        return combine_splitk(y, group=group, inplace=True)
    return gather_rows(y, group=group) if gather and G > 1 else y
