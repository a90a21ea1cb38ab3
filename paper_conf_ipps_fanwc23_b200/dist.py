"""Multi-GPU host logic: nnz-balanced shards and the X all-gather.

SpMM is sharded by contiguous rows with equal nnz (gnn_shard_rows), SDDMM by equal edge
ranges (gnn_shard_edges); each rank plans and runs its shard on zero-copy sub-views and
keeps its outputs.  The only exchange is the feature matrix X: replicated, or
all-gathered as equal padded row blocks (NCCL all_gather_into_tensor over NVLink).
The paper itself is single-GPU; this layer is the BJ "1/2/4/8 B200" extension.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np
import torch
import torch.distributed as dist

from . import DeviceGraph, shard_edges, shard_rows


@dataclass(frozen=True)
class ShardSpec:
    rank: int
    world: int
    r0: int  # SpMM rows [r0, r1) ...
    r1: int
    e0: int  # ... whose nnz are [e0, e1)
    e1: int
    f0: int  # SDDMM edges [f0, f1)
    f1: int
    xblk: int  # rows of X owned per rank for the all-gather (ceil(N / world))
    x0: int    # this rank's owned X rows [x0, x1)
    x1: int


def shard_spec(row_ptr: np.ndarray, N: int, rank: int, world: int) -> ShardSpec:
    """Shard bounds for `rank` of `world` (host only; identical on every rank)."""
    rb = shard_rows(row_ptr, world)
    nnz = int(row_ptr[-1]) - int(row_ptr[0])
    eb = shard_edges(nnz, world)
    r0, r1 = int(rb[rank]), int(rb[rank + 1])
    base = int(row_ptr[0])
    blk = -(-N // world) if N else 0
    x0 = min(N, rank * blk)
    x1 = min(N, x0 + blk)
    return ShardSpec(rank, world, r0, r1, int(row_ptr[r0]) - base, int(row_ptr[r1]) - base,
                     int(eb[rank]), int(eb[rank + 1]), blk, x0, x1)


def local_graphs(full: DeviceGraph, s: ShardSpec):
    """(SpMM row-shard view, SDDMM edge-shard view) of a resident full graph."""
    if s.world == 1:
        return full, full
    sp = full.shard(s.r0, s.r1, s.e0, s.e1)
    sd = DeviceGraph(full.M, full.N, full.row_ind[s.f0:s.f1], full.col_ind[s.f0:s.f1],
                     None if full.val is None else full.val[s.f0:s.f1], None, full.row_base)
    return sp, sd


def gather_features(own: torch.Tensor, s: ShardSpec, N: int, out: torch.Tensor | None = None,
                    group=None) -> torch.Tensor:
    """All-gather the row blocks of X (each rank owns rows [x0, x1), padded to xblk rows)
    into an (xblk * world) x K tensor whose first N rows are X."""
    K = own.shape[1]
    if own.shape[0] != s.xblk:
        pad = torch.zeros((s.xblk, K), dtype=own.dtype, device=own.device)
        pad[:own.shape[0]] = own
        own = pad
    if out is None:
        out = torch.empty((s.xblk * s.world, K), dtype=own.dtype, device=own.device)
    dist.all_gather_into_tensor(out, own.contiguous(), group=group)
    return out


# ------------------------------------------------------------------------------
# f1: overlap the X all-gather with SpMM.  Each rank splits its row shard
# by column owner block (gnn_split_col_blocks), computes the block whose X rows it owns
# while the other blocks are still being broadcast, then each remaining block as soon as
# its broadcast lands, accumulating into O (gnn_spmm_ex with beta = 1) in a fixed order.

def block_order(P: int, p: int):
    """Compute order on rank p: the local block first, then the others in the order
    their broadcasts are issued (0..P-1, skipping p)."""
    return [p] + [q for q in range(P) if q != p]


def start_block_broadcasts(X_full: torch.Tensor, s: ShardSpec, group=None):
    """Issue one broadcast per owner block (the same order on every rank) and return the
    async works; works[q].wait() makes the current stream wait for block q."""
    works = []
    for q in range(s.world):
        blk = X_full[q * s.xblk:(q + 1) * s.xblk]
        works.append(dist.broadcast(blk, src=q, group=group, async_op=True))
    return works


class OverlappedSpMM:
    """Row-shard SpMM whose feature rows arrive block by block (f1)."""

    def __init__(self, row_ind, col_ind, val, s: ShardSpec, K: int, device, group=None):
        from . import DeviceGraph, plan, split_col_blocks
        import numpy as _np
        self.s, self.K, self.group = s, K, group
        ro, co, vo, b = split_col_blocks(_np.asarray(row_ind)[s.e0:s.e1],
                                         _np.asarray(col_ind)[s.e0:s.e1],
                                         None if val is None else _np.asarray(val)[s.e0:s.e1],
                                         s.world, s.xblk)
        self.bounds = b
        t = lambda a, dt: torch.from_numpy(a).to(device=device, dtype=dt)
        self.ri, self.ci = t(ro, torch.int32), t(co, torch.int32)
        self.vi = None if vo is None else t(vo, torch.float32)
        self.blocks, self.plans = [], []
        for q in range(s.world):
            a, z = int(b[q]), int(b[q + 1])
            g = DeviceGraph(s.r1 - s.r0, s.xblk * s.world, self.ri[a:z], self.ci[a:z],
                            None if self.vi is None else self.vi[a:z], None, s.r0)
            self.blocks.append(g)
            self.plans.append(plan(g, K))
        self.X_full = torch.empty((s.xblk * s.world, K), dtype=torch.float32, device=device)

    def __call__(self, X_own: torch.Tensor, O: torch.Tensor, replan: bool = True) -> torch.Tensor:
        """X_own: this rank's xblk x K rows (padded); O: (r1 - r0) x K output.  Returns
        the gathered X (complete on the current stream when this returns).  replan=True
        rebuilds the per-block plans (GPU plan kernel) as part of the step."""
        from . import plan, spmm
        s = self.s
        if replan:
            self.plans = [plan(g, self.K) for g in self.blocks]
        self.X_full[s.rank * s.xblk:(s.rank + 1) * s.xblk].copy_(X_own)
        works = start_block_broadcasts(self.X_full, s, self.group)
        first = True
        for q in block_order(s.world, s.rank):
            if q != s.rank:
                works[q].wait()
            spmm(self.plans[q], self.blocks[q], self.X_full, out=O, accumulate=not first)
            first = False
        return self.X_full
