"""Autograd and a GCN layer on the C ABI.

The paper's end goal is GNN training (Table V): a GCN layer is "an SpMM
operation followed by a fully-connected layer".  This module wires the library's
SpMM / SDDMM into torch.autograd:

    O = (+)_{i: row_i = r} v_i X[col_i]           forward   (gnn_spmm / gnn_spmm_ex)
    dX = S^T dO  (mean: S^T (dO / cnt))           backward  (gnn_spmm on gnn_transpose(S))
    dv_i = <dO[row_i], X[col_i]>                  backward  (gnn_sddmm: SDDMM is the
                                                             gradient of SpMM w.r.t. v)

    max / min: the first nonzero of each row attaining the extremum takes the gradient
    of each (row, column)                               (gnn_spmm_extremum_backward)
All arithmetic runs in the library's kernels; torch supplies memory and the dense GEMM of
the fully-connected part (cuBLAS, a plain library GEMM).
"""
from __future__ import annotations

import math

import torch

from . import (DeviceGraph, gather_values, plan, scale_rows_inv_degree, sddmm, spmm,
               spmm_extremum_backward, transpose)


class SparseOp:
    """A graph prepared for training: S on the device, S^T (built once by gnn_transpose)
    and cached plans per (direction, K, feature dtype)."""

    def __init__(self, graph: DeviceGraph, need_transpose: bool = True):
        self.g = graph
        self.gt, self.perm = (transpose(graph) if need_transpose else (None, None))
        self._plans = {}

    def plan_for(self, which: str, K: int, dtype=torch.float32):
        key = (which, K, dtype)
        p = self._plans.get(key)
        if p is None:
            p = plan(self.g if which == "f" else self.gt, K, feature_dtype=dtype)
            self._plans[key] = p
        return p

    def with_val(self, val, transposed=False) -> DeviceGraph:
        g = self.gt if transposed else self.g
        if val is not None and transposed:  # S^T's values in transposed order (edge_perm)
            val = gather_values(val.contiguous(), self.perm)
        return DeviceGraph(g.M, g.N, g.row_ind, g.col_ind, val, g.row_ptr, g.row_base)


class _SpMMFunction(torch.autograd.Function):
    @staticmethod
    def forward(ctx, X, val, op: SparseOp, agg: str):
        X = X.contiguous()
        K = X.shape[1]
        g = op.g if val is None else op.with_val(val.detach().contiguous())
        O = spmm(op.plan_for("f", K, X.dtype), g, X, agg=agg)
        ctx.op, ctx.agg = op, agg
        ctx.save_for_backward(X, val, O if agg in ("max", "min") else None)
        return O

    @staticmethod
    def backward(ctx, dO):
        X, val, O = ctx.saved_tensors
        op, agg = ctx.op, ctx.agg
        dO = dO.contiguous().float()
        if agg in ("max", "min"):
            if X.dtype != torch.float32:
                raise NotImplementedError("max / min backward: fp32 features only")
            g = op.g if val is None else op.with_val(val.detach().contiguous())
            need_v = val is not None and ctx.needs_input_grad[1]
            dval = torch.zeros(op.g.nnz, dtype=torch.float32, device=X.device) if need_v else None
            dX, dval = spmm_extremum_backward(g, agg, X, O, dO, dval=dval)
            return (dX if ctx.needs_input_grad[0] else None), dval, None, None
        if agg == "mean":  # dX = S^T (dO / deg): the row scale runs in the library
            dO = scale_rows_inv_degree(op.g, dO)
        K = dO.shape[1]
        dX = dval = None
        if ctx.needs_input_grad[0]:
            if op.gt is None:
                raise RuntimeError("SparseOp was built without the transpose")
            gt = op.gt if val is None else op.with_val(val.detach(), transposed=True)
            dX = spmm(op.plan_for("t", K), gt, dO).to(X.dtype)
        if val is not None and ctx.needs_input_grad[1]:
            g1 = DeviceGraph(op.g.M, op.g.N, op.g.row_ind, op.g.col_ind, None, op.g.row_ptr,
                             op.g.row_base)
            dval = sddmm(op.plan_for("f", K), g1, dO, X.float())
        return dX, dval, None, None


def spmm_autograd(op: SparseOp, X: torch.Tensor, val: torch.Tensor | None = None,
                  agg: str = "sum") -> torch.Tensor:
    """Differentiable O = S X (or the mean aggregation); gradients for X and, when val
    is given and requires grad, for the edge values."""
    return _SpMMFunction.apply(X, val, op, agg)


class GCNConv(torch.nn.Module):
    """H' = S (H W) + b  (GCN layer: SpMM after the fully-connected transform)."""

    def __init__(self, fin: int, fout: int, bias: bool = True, agg: str = "sum"):
        super().__init__()
        self.weight = torch.nn.Parameter(torch.empty(fin, fout))
        self.bias = torch.nn.Parameter(torch.zeros(fout)) if bias else None
        self.agg = agg
        bound = math.sqrt(6.0 / (fin + fout))
        torch.nn.init.uniform_(self.weight, -bound, bound)

    def forward(self, op: SparseOp, H: torch.Tensor) -> torch.Tensor:
        out = spmm_autograd(op, H @ self.weight, agg=self.agg)
        return out + self.bias if self.bias is not None else out


class GCN(torch.nn.Module):
    def __init__(self, fin: int, hidden: int, classes: int, layers: int = 2):
        super().__init__()
        dims = [fin] + [hidden] * (layers - 1) + [classes]
        self.convs = torch.nn.ModuleList(GCNConv(a, b) for a, b in zip(dims, dims[1:]))

    def forward(self, op: SparseOp, H: torch.Tensor) -> torch.Tensor:
        for i, conv in enumerate(self.convs):
            H = conv(op, H)
            if i + 1 < len(self.convs):
                H = torch.relu(H)
        return H
