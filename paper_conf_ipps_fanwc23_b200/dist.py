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
