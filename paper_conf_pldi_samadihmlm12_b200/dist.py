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

The local computations are the C-ABI kernels (``ops.mv/tmv/dot``); ``local_fn``
and ``merge_fn`` hooks exist only so the host logic can be exercised on CPU
with the gloo backend in tests.
"""
from __future__ import annotations

from typing import Callable, Optional

import torch
import torch.distributed as dist

from . import ops


def shard_range(n: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous block partition of [0, n): the first n % world ranks get one extra."""
    if world <= 0 or not 0 <= rank < world or n < 0:
        raise ValueError("bad shard arguments")
    base, rem = divmod(n, world)
    start = rank * base + min(rank, rem)
    return start, start + base + (1 if rank < rem else 0)


def _world(group):
    return dist.get_world_size(group), dist.get_rank(group)


def mv_rowshard(A_local: torch.Tensor, x: torch.Tensor, *, group=None, gather: bool = False,
                local_fn: Optional[Callable] = None, variant="AUTO") -> torch.Tensor:
    """y rows of this rank's A block (R_local x C); optionally all-gathered to the full y.
    With gather=True every rank must hold shard_range-sized blocks."""
    fn = local_fn or (lambda A, xx: ops.mv(A, xx, variant=variant))
    y_local = fn(A_local, x)
    if not gather:
        return y_local
    G, _ = _world(group)
    sizes = [None] * G
    dist.all_gather_object(sizes, int(y_local.numel()), group=group)
    width = max(sizes)                  # collectives need equal sizes: pad, gather, trim
    padded = torch.zeros(width, dtype=y_local.dtype, device=y_local.device)
    padded[: y_local.numel()] = y_local
    parts = [torch.empty(width, dtype=y_local.dtype, device=y_local.device) for _ in sizes]
    dist.all_gather(parts, padded, group=group)
    return torch.cat([p[:s] for p, s in zip(parts, sizes)])


def combine_splitk(y_part: torch.Tensor, *, group=None,
                   merge_fn: Optional[Callable] = None) -> torch.Tensor:
    """Combine per-rank partial sums of the same R outputs into the full y (every rank)."""
    if y_part.dtype == torch.float32:
        y = y_part.clone()
        dist.all_reduce(y, op=dist.ReduceOp.SUM, group=group)
        return y
    if y_part.dtype != torch.int32:
        raise TypeError("split-K combine supports float32 and int32")
    G, _ = _world(group)
    P = torch.empty(G, y_part.numel(), dtype=torch.int32, device=y_part.device)
    dist.all_gather(list(P.unbind(0)), y_part.contiguous().view(-1), group=group)
    if merge_fn is not None:
        return merge_fn(P)
    ones = torch.ones(G, dtype=torch.int32, device=P.device)
    return ops.tmv(P, ones)          # y[r] = sum_g P[g, r] (mod 2^32), fixed order


def tmv_splitk(B_local: torch.Tensor, x_local: torch.Tensor, *, group=None,
               local_fn: Optional[Callable] = None, merge_fn: Optional[Callable] = None,
               variant="AUTO") -> torch.Tensor:
    """B_local: this rank's contiguous rows [c0, c1) of the C x R matrix B; x_local = x[c0:c1].
    Returns the full y (R outputs) on every rank."""
    fn = local_fn or (lambda B, xx: ops.tmv(B, xx, variant=variant))
    return combine_splitk(fn(B_local, x_local), group=group, merge_fn=merge_fn)


def mv_splitk(A_local: torch.Tensor, x_local: torch.Tensor, *, group=None,
              local_fn: Optional[Callable] = None, merge_fn: Optional[Callable] = None,
              variant="AUTO") -> torch.Tensor:
    """A_local: this rank's column block of A, stored as its own R x C_local array."""
    fn = local_fn or (lambda A, xx: ops.mv(A, xx, variant=variant))
    return combine_splitk(fn(A_local, x_local), group=group, merge_fn=merge_fn)


def dot_splitk(a_local: torch.Tensor, b_local: torch.Tensor, *, group=None,
               local_fn: Optional[Callable] = None, merge_fn: Optional[Callable] = None,
               variant="AUTO") -> torch.Tensor:
    """Fewer pairs than ranks (e.g. Sdot, N = 1): split each pair's length."""
    fn = local_fn or (lambda a, b: ops.dot(a, b, variant=variant))
    return combine_splitk(fn(a_local, b_local), group=group, merge_fn=merge_fn)
