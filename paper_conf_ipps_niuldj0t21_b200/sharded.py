"""Tile-row sharding of the tiled SpMV over the GPUs of one node.

Rows are independent in SpMV (Alg. 1), and the 16-row tile
row is the method's natural unit, so rank r owns a contiguous range of
tile rows, builds its own tiled matrix from that row slice (global column
space, x replicated), computes its y rows, and an all-gather of y over
NCCL/NVLink assembles the next iterate on every rank.  Because the SpMV work
items depend only on a tile row's own content, every row is summed in the same
order as on one GPU and the gathered vector equals the 1-GPU y bitwise.

The collective is torch.distributed (backend "nccl" on B200s, "gloo" in the
CPU tests); `spmv` is any callable (x_full, y_out) -> None, normally
TiledMatrix.run.
"""
from __future__ import annotations

import numpy as np


def partition_tile_rows(nrows: int, P: int, weights=None) -> list[int]:
    """P+1 row boundaries, each a multiple of 16 except the last (= nrows),
    splitting the ceil(nrows/16) tile rows into P contiguous ranges balanced
    by `weights` (one non-negative number per tile row) or by count."""
    T = (nrows + 15) // 16
    if P <= 1:
        return [0, nrows]
    if weights is None:
        cuts = [(T * r) // P for r in range(P + 1)]
    else:
        w = np.asarray(weights, dtype=np.float64)
        assert w.shape == (T,)
        c = np.concatenate([[0.0], np.cumsum(w + 1e-9)])  # +eps: empty rows still count
        tot = c[-1]
        cuts = [0] + [int(np.searchsorted(c, tot * r / P, side="left")) for r in range(1, P)] + [T]
        for r in range(1, P + 1):  # monotone
            cuts[r] = max(cuts[r], cuts[r - 1])
    return [min(16 * t, nrows) for t in cuts[:-1]] + [nrows]


class ShardedSpMV:
    """One rank's side of the sharded iterated SpMV x_{k+1} = A x_k."""

    def __init__(self, spmv, bounds: list[int], rank: int, world: int, group=None, device=None,
                 dtype=None):
        import torch
        self.spmv = spmv
        self.bounds = bounds
        self.rank, self.world, self.group = rank, world, group
        self.rows = bounds[rank + 1] - bounds[rank]
        self.maxrows = max(bounds[i + 1] - bounds[i] for i in range(world))
        self.m = bounds[-1]
        self.equal = all(bounds[i + 1] - bounds[i] == self.maxrows for i in range(world))
        dtype = dtype or torch.float64
        # padded gather buffer; rank r's y rows live at [r*maxrows, r*maxrows + rows)
        self.gathered = torch.zeros(world * self.maxrows, dtype=dtype, device=device)

    def local_out(self):
        b = self.rank * self.maxrows
        return self.gathered[b:b + self.rows]

    def step(self, x_full, x_next=None):
        """y_local = A_local x_full, then all-gather into x_next (length m)."""
        import torch
        import torch.distributed as dist
        self.spmv(x_full, self.local_out())
        chunk = self.gathered[self.rank * self.maxrows:(self.rank + 1) * self.maxrows]
        if self.world > 1:
            dist.all_gather_into_tensor(self.gathered, chunk, group=self.group)
        if self.equal and x_next is None:
            return self.gathered[:self.m]
        if x_next is None:
            x_next = torch.empty(self.m, dtype=self.gathered.dtype, device=self.gathered.device)
        for r in range(self.world):
            a, b = self.bounds[r], self.bounds[r + 1]
            x_next[a:b].copy_(self.gathered[r * self.maxrows:r * self.maxrows + (b - a)])
        return x_next
