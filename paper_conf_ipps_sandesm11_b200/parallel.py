"""Multi-GPU column-stripe pipeline -- host side.

One process per GPU (torchrun).  Rank g owns global columns
[floor(g n / P), floor((g+1) n / P)) of S1 and sweeps every band of them; the
kernel hands each band's right-edge column (t, E) to rank g+1 by peer stores
into rank g+1's receive area (a CUDA IPC mapping over NVLink), guarded by
per-(band, warp) epoch flags.  This module only does plumbing:

- ``stripe_bounds``: the partition (pure);
- ``combine_best``: the (score, min i, min j) order across ranks (pure);
- ``StripeGroup``: exchanges the receive-area IPC handles through
  ``torch.distributed`` (any backend with object collectives), keeps the
  epoch counter in lock-step, runs the rank's stripe and combines the bests.

No data-path collective is used: the only exchange on the hot path is the
kernel's own border hand-off.
"""
from __future__ import annotations

from typing import Iterable, Optional, Sequence, Tuple


def stripe_bounds(n: int, world: int, rank: int) -> Tuple[int, int]:
    """Global 0-based column range [c_lo, c_hi) of `rank` among `world` stripes."""
    if world < 1 or not (0 <= rank < world):
        raise ValueError("bad rank/world")
    if n < world:
        raise ValueError(f"n={n} columns cannot be split into {world} non-empty stripes")
    return (n * rank) // world, (n * (rank + 1)) // world


def combine_best(results: Iterable[Sequence[int]]) -> Tuple[int, int, int]:
    """Best (score, i, j) under the library's total order (sw_combine_best:
    higher score, then smaller i, then smaller j; (0, 0, 0) when every score
    is 0, reading S4).  Marshalling only."""
    from . import combine_best as _lib_combine

    return _lib_combine(results)


def exchange_handles(my_handle: Optional[bytes], rank: int, world: int, group=None) -> Optional[bytes]:
    """All-gather the 64-byte receive-area handles; return the right neighbour's
    (None for the last rank)."""
    import torch.distributed as dist

    handles = [None] * world
    dist.all_gather_object(handles, my_handle, group=group)
    return handles[rank + 1] if rank + 1 < world else None


class StripeGroup:
    """This rank's stripe of a multi-GPU Stage 1 (see module docstring)."""

    def __init__(self, ctx, rank: int, world: int, max_rows: int, group=None):
        import torch.distributed as dist

        self.ctx, self.rank, self.world, self.group = ctx, rank, world, group
        self.max_rows = max_rows
        my = ctx.stripe_export(max_rows) if rank > 0 else None
        right = exchange_handles(my, rank, world, group)
        ctx.stripe_connect(right, max_rows)
        dist.barrier(group=group)

    def _agree(self, value):
        import torch.distributed as dist

        vals = [None] * self.world
        dist.all_gather_object(vals, value, group=self.group)
        return vals

    def align_stage1(self, dA_ptr: int, m: int, dB_ptr: int, n: int, scoring=(1, -3, 3, 2), k: int = 0,
                     sink=None, stream: int = 0):
        """Run this rank's stripe; returns (global best, local best, (c_lo, c_hi)).
        `sink(row, H_slice, F_slice)` receives this stripe's slice of each special row."""
        if m > self.max_rows:
            raise ValueError("m exceeds the receive area")
        c_lo, c_hi = stripe_bounds(n, self.world, self.rank)
        # the epoch: above every epoch any rank's receive area has seen (the flags
        # are compared for equality), the same on all ranks
        plan = self.ctx.plan(m, n, *scoring, k=k, world=0)
        info = self._agree((self.ctx.stripe_epoch(), plan))
        if len({p for _, p in info}) != 1:
            raise RuntimeError(f"ranks chose different kernel geometries {[p for _, p in info]}: the band "
                               f"height must agree (same library build, GPU and overrides)")
        epoch = 1 + max(e for e, _ in info)
        local, _ = self.ctx.align_stage1_stripe(dA_ptr, m, dB_ptr, n, c_lo, c_hi, epoch, *scoring, k=k,
                                                sink=sink, stream=stream)
        allres = self._agree(local.astuple())
        return combine_best(allres), local.astuple(), (c_lo, c_hi)


class CyclicGroup:
    """This rank's share of a band-cyclic multi-GPU Stage 1:
    rank r runs bands r, r + world, ...; each band's bottom row and progress go
    to rank (r + 1) mod world by peer stores into its CUDA IPC area.  The
    handles are exchanged here; the epoch and the kernel geometry are agreed
    before each call; the ranks' bests are combined by the library's order."""

    def __init__(self, ctx, rank: int, world: int, max_rows: int, max_cols: int, group=None):
        import torch.distributed as dist

        if world < 2:
            raise ValueError("a band-cyclic group needs at least two ranks")
        self.ctx, self.rank, self.world, self.group = ctx, rank, world, group
        self.max_rows, self.max_cols = max_rows, max_cols
        mine = ctx.cyclic_export(max_rows, max_cols)
        handles = [None] * world
        dist.all_gather_object(handles, mine, group=group)
        ctx.cyclic_connect(handles[(rank + 1) % world], max_rows, max_cols)
        dist.barrier(group=group)

    def _agree(self, value):
        import torch.distributed as dist

        vals = [None] * self.world
        dist.all_gather_object(vals, value, group=self.group)
        return vals

    def align_stage1(self, dA_ptr: int, m: int, dB_ptr: int, n: int, scoring=(1, -3, 3, 2), k: int = 0,
                     sink=None, stream: int = 0):
        """Run this rank's bands; returns (global best, local best).  `sink(row, H, F)`
        receives the whole special rows of this rank's bands."""
        if m > self.max_rows or n > self.max_cols:
            raise ValueError("the matrix exceeds the band-cyclic areas")
        plan = self.ctx.plan(m, n, *scoring, k=k, world=self.world)
        info = self._agree((self.ctx.cyclic_epoch(), plan))
        if len({p for _, p in info}) != 1:
            raise RuntimeError(f"ranks chose different kernel geometries {[p for _, p in info]}")
        epoch = 1 + max(e for e, _ in info)
        local, _ = self.ctx.align_stage1_cyclic(dA_ptr, m, dB_ptr, n, self.rank, self.world, epoch, *scoring, k=k,
                                                sink=sink, stream=stream)
        return combine_best(self._agree(local.astuple())), local.astuple()
