"""Thin Python binding of libgnnsparse.so (the C ABI in include/gnn_sparse.h).

Hybrid-parallel SpMM / SDDMM for GNN message passing on B200 (sm_100a), after
Fan, Wang, Chu, IPDPS 2023.  This module only marshals arguments:
every step of the hot path (plan, SpMM, SDDMM) runs in the library's CUDA kernels.
PyTorch provides device memory, streams and process groups.  There is no CPU
fallback: if the shared library or a CUDA device is missing, calls raise.

Names follow the C ABI: ``plan`` (gnn_plan_create), ``spmm`` (gnn_spmm),
``sddmm`` (gnn_sddmm), ``shard_rows`` / ``shard_edges``, ``csr_to_coo``,
``validate``.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field

import numpy as np
import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
# GNN_LIB_PATH selects an alternative in-tree build (tuning sweeps, tools/sweep.py)
LIB_PATH = os.environ.get("GNN_LIB_PATH", os.path.join(_HERE, "libgnnsparse.so"))

__all__ = ["DeviceGraph", "Plan", "PlanOpts", "plan", "spmm", "sddmm", "shard_rows",
           "shard_edges", "reorder_gcr", "permute_graph", "permute_rows", "csr_to_coo",
           "validate", "GnnError", "lib", "LIB_PATH"]

GNN_OK, GNN_ERR_INVALID_ARG, GNN_ERR_UNSUPPORTED, GNN_ERR_CUDA, GNN_ERR_WORKSPACE, \
    GNN_ERR_INPUT_CHECK = range(6)


class GnnError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"[gnn status {status}] {msg}")
        self.status = status


class _Graph(ctypes.Structure):
    _fields_ = [("M", ctypes.c_int64), ("N", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("row_ptr", ctypes.c_void_p), ("row_ind", ctypes.c_void_p),
                ("col_ind", ctypes.c_void_p), ("val", ctypes.c_void_p),
                ("row_base", ctypes.c_int64)]


class PlanOpts(ctypes.Structure):
    """gnn_plan_opts_t; zero fields take the library defaults (alpha 2, 2 warps/block)."""
    _fields_ = [("alpha", ctypes.c_int32), ("warps_per_block", ctypes.c_int32),
                ("force_chunk", ctypes.c_int32), ("force_vw", ctypes.c_int32),
                ("deterministic", ctypes.c_int32), ("feature_dtype", ctypes.c_int32),
                ("no_locality", ctypes.c_int32), ("num_sms", ctypes.c_int32),
                ("active_blocks_per_sm", ctypes.c_int32), ("l2_bytes", ctypes.c_int64)]


class _PlanInfo(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in (
        "chunk", "vw_feat", "vw_sparse", "lanes", "vecs", "slices", "groups", "warps_per_block",
        "active_blocks_per_sm", "num_sms", "alpha", "K", "feature_dtype", "chunk_dtp")] + [
        ("nnz", ctypes.c_int64), ("num_chunks", ctypes.c_int64), ("num_blocks", ctypes.c_int64),
        ("M", ctypes.c_int64), ("l2_bytes", ctypes.c_int64)]


class ReorderOpts(ctypes.Structure):
    """gnn_reorder_opts_t; zero fields take defaults (3 levels, 20 passes, 1e-6, 1.0)."""
    _fields_ = [("max_levels", ctypes.c_int32), ("max_passes", ctypes.c_int32),
                ("min_gain", ctypes.c_double), ("resolution", ctypes.c_double),
                ("hub_rows", ctypes.c_int64)]


EXPORTS = ["gnn_plan_workspace_bytes", "gnn_plan_create", "gnn_plan_info", "gnn_plan_arrays",
           "gnn_plan_destroy", "gnn_spmm", "gnn_sddmm", "gnn_spmm_bf16", "gnn_sddmm_bf16",
           "gnn_spmm_ex", "gnn_spmm_extremum_backward", "gnn_plan_spmm_sddmm",
           "gnn_transpose_workspace_bytes",
           "gnn_transpose", "gnn_gather_f32", "gnn_scale_rows_inv_degree",
           "gnn_shard_rows", "gnn_shard_edges", "gnn_split_col_blocks",
           "gnn_reorder_gcr", "gnn_permute_graph", "gnn_permute_rows",
           "gnn_probe_gather", "gnn_probe_gather_chunked", "gnn_run_host_workspace_bytes", "gnn_run_host",
           "gnn_run_host_multi_workspace_bytes", "gnn_run_host_multi", "gnn_csr_to_coo", "gnn_validate", "gnn_last_error",
           "gnn_version"]

_lib = None


def lib():
    """Load libgnnsparse.so (raises if it has not been built -- no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} missing: run `make` (or __graft_entry__.build()) first")
    L = ctypes.CDLL(LIB_PATH)
    vp, i64, i32, st = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_int
    P = ctypes.POINTER
    L.gnn_plan_workspace_bytes.argtypes = [i64, i64, i32, P(PlanOpts)]
    L.gnn_plan_workspace_bytes.restype = ctypes.c_size_t
    L.gnn_plan_create.argtypes = [P(_Graph), i32, P(PlanOpts), vp, ctypes.c_size_t, vp, P(vp)]
    L.gnn_plan_info.argtypes = [vp, P(_PlanInfo)]
    L.gnn_plan_arrays.argtypes = [vp, P(vp), P(vp), P(vp)]
    L.gnn_plan_destroy.argtypes = [vp]
    L.gnn_plan_destroy.restype = None
    L.gnn_spmm.argtypes = [vp, P(_Graph), vp, i64, vp, i64, vp]
    L.gnn_sddmm.argtypes = [vp, P(_Graph), vp, i64, vp, i64, vp, vp]
    if hasattr(L, "gnn_spmm_bf16"):  # (GNN_LIB_PATH may point at an older tuning build)
        L.gnn_spmm_bf16.argtypes = [vp, P(_Graph), vp, i64, vp, i64, vp]
        L.gnn_sddmm_bf16.argtypes = [vp, P(_Graph), vp, i64, vp, i64, vp, vp]
    if hasattr(L, "gnn_spmm_ex"):
        L.gnn_spmm_ex.argtypes = [vp, P(_Graph), vp, i64, vp, i64, i32, i32, vp]
        L.gnn_spmm_extremum_backward.argtypes = [P(_Graph), i32, i32, vp, i64, vp, i64, vp,
                                                 i64, vp, i64, vp, vp]
        L.gnn_plan_spmm_sddmm.argtypes = [P(_Graph), i32, P(PlanOpts), vp, i64, vp, i64, vp, vp,
                                          ctypes.c_size_t, vp]
        L.gnn_transpose_workspace_bytes.argtypes = [i64]
        L.gnn_transpose_workspace_bytes.restype = ctypes.c_size_t
        L.gnn_transpose.argtypes = [P(_Graph), vp, ctypes.c_size_t, vp, vp, vp, vp, vp, vp]
    if hasattr(L, "gnn_gather_f32"):
        L.gnn_gather_f32.argtypes = [vp, vp, i64, vp, vp]
        L.gnn_scale_rows_inv_degree.argtypes = [vp, i64, i32, vp, i64, vp, i64, vp]
    L.gnn_shard_rows.argtypes = [vp, i64, i32, vp]
    L.gnn_shard_edges.argtypes = [i64, i32, vp]
    if hasattr(L, "gnn_run_host"):
        L.gnn_run_host_workspace_bytes.argtypes = [i64, i64, i64, i32, P(PlanOpts)]
        L.gnn_run_host_workspace_bytes.restype = ctypes.c_size_t
        if hasattr(L, "gnn_run_host_multi"):  # (GNN_LIB_PATH may point at an older build)
            L.gnn_run_host_multi_workspace_bytes.argtypes = [i64, i64, i64, i32, vp,
                                                             P(PlanOpts)]
            L.gnn_run_host_multi_workspace_bytes.restype = ctypes.c_size_t
            L.gnn_run_host_multi.argtypes = [P(_Graph), i32, i32, vp, vp, vp, vp, P(PlanOpts),
                                             vp, ctypes.c_size_t, vp]
        L.gnn_run_host.argtypes = [P(_Graph), i32, vp, i32, vp, vp, P(PlanOpts), vp,
                                   ctypes.c_size_t, vp]
    if hasattr(L, "gnn_split_col_blocks"):
        L.gnn_split_col_blocks.argtypes = [vp, vp, vp, i64, i32, i64, vp, vp, vp, vp]
    L.gnn_csr_to_coo.argtypes = [vp, i64, i64, vp, vp]
    L.gnn_reorder_gcr.argtypes = [vp, vp, i64, P(ReorderOpts), vp, vp, P(ctypes.c_double)]
    L.gnn_permute_graph.argtypes = [vp, vp, vp, i64, vp, vp, vp, vp, vp]
    L.gnn_permute_rows.argtypes = [vp, i64, i64, i64, vp, vp, i64, vp]
    L.gnn_probe_gather.argtypes = [vp, i64, vp, i64, i32, vp, vp]
    if hasattr(L, "gnn_probe_gather_chunked"):
        L.gnn_probe_gather_chunked.argtypes = [vp, i64, vp, i64, i32, i32, vp, vp]
    L.gnn_validate.argtypes = [P(_Graph), vp]
    L.gnn_last_error.argtypes = []
    L.gnn_last_error.restype = ctypes.c_char_p
    L.gnn_version.argtypes = []
    L.gnn_version.restype = ctypes.c_char_p
    for f in ("gnn_plan_create", "gnn_plan_info", "gnn_plan_arrays", "gnn_spmm", "gnn_sddmm",
              "gnn_shard_rows", "gnn_shard_edges", "gnn_csr_to_coo", "gnn_validate",
              "gnn_reorder_gcr", "gnn_permute_graph", "gnn_permute_rows", "gnn_probe_gather",
              "gnn_probe_gather_chunked",
              "gnn_spmm_bf16", "gnn_sddmm_bf16", "gnn_spmm_ex", "gnn_transpose",
              "gnn_split_col_blocks", "gnn_run_host", "gnn_run_host_multi", "gnn_gather_f32",
              "gnn_scale_rows_inv_degree"):
        if hasattr(L, f):
            getattr(L, f).restype = st
    _lib = L
    return L


def _check(status):
    if status != GNN_OK:
        raise GnnError(status, lib().gnn_last_error().decode())


def _stream(stream=None):
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def _ptr(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


# ----------------------------------------------------------------- graph ----
@dataclass
class DeviceGraph:
    """Hybrid CSR/COO adjacency resident on a CUDA device.
    row_ind is the decoded, non-decreasing row index; val None means all ones.
    A row shard keeps global row ids in [row_base, row_base + M)."""
    M: int
    N: int
    row_ind: torch.Tensor
    col_ind: torch.Tensor
    val: torch.Tensor | None = None
    row_ptr: torch.Tensor | None = None
    row_base: int = 0
    _keep: list = field(default_factory=list, repr=False)

    @property
    def nnz(self) -> int:
        return int(self.row_ind.numel())

    @staticmethod
    def from_arrays(M, N, row_ind, col_ind, val=None, row_ptr=None, device="cuda",
                    row_base=0):
        def dev(a, dt):
            if a is None:
                return None
            t = torch.as_tensor(np.asarray(a) if not torch.is_tensor(a) else a)
            return t.to(device=device, dtype=dt).contiguous()
        return DeviceGraph(int(M), int(N), dev(row_ind, torch.int32), dev(col_ind, torch.int32),
                           dev(val, torch.float32), dev(row_ptr, torch.int32), int(row_base))

    def shard(self, r0: int, r1: int, e0: int, e1: int) -> "DeviceGraph":
        """Zero-copy view of rows [r0, r1) whose nnz are [e0, e1) (a row shard)."""
        return DeviceGraph(r1 - r0, self.N, self.row_ind[e0:e1], self.col_ind[e0:e1],
                           None if self.val is None else self.val[e0:e1],
                           None if self.row_ptr is None else self.row_ptr[r0:r1 + 1],
                           self.row_base + r0)

    def desc(self) -> _Graph:
        # cached: the descriptor is rebuilt only if an array was replaced
        key = (self.M, self.N, self.row_base,
               *(None if t is None else (t.data_ptr(), t.numel())
                 for t in (self.row_ptr, self.row_ind, self.col_ind, self.val)))
        if self._keep and self._keep[0] == key:
            return self._keep[1]
        d = _Graph(self.M, self.N, self.nnz, _ptr(self.row_ptr), _ptr(self.row_ind),
                   _ptr(self.col_ind), _ptr(self.val), self.row_base)
        self._keep[:] = [key, d]
        return d


# ------------------------------------------------------------------ plan ----
class Plan:
    """Owns the plan handle and its device workspace (a torch uint8 tensor)."""

    def __init__(self, handle, workspace, graph, K):
        self._h = handle
        self.workspace = workspace
        self.graph = graph
        self.K = K

    @property
    def handle(self):
        return self._h

    def info(self) -> dict:
        inf = _PlanInfo()
        _check(lib().gnn_plan_info(self._h, ctypes.byref(inf)))
        return {n: getattr(inf, n) for n, _ in _PlanInfo._fields_}

    def arrays(self):
        """(row_first, row_last, flags) as device tensors (views into the workspace)."""
        rf, rl, fl = ctypes.c_void_p(), ctypes.c_void_p(), ctypes.c_void_p()
        _check(lib().gnn_plan_arrays(self._h, ctypes.byref(rf), ctypes.byref(rl),
                                     ctypes.byref(fl)))
        nch = self.info()["num_chunks"]
        if nch == 0:
            z = torch.empty(0, dtype=torch.int32, device=self.workspace.device)
            return z, z.clone(), torch.empty(0, dtype=torch.uint8, device=z.device)
        base = self.workspace.data_ptr()
        ws = self.workspace
        def view(ptr, nbytes, dt):
            off = ptr - base
            return ws[off:off + nbytes].view(dt)
        return (view(rf.value, 4 * nch, torch.int32), view(rl.value, 4 * nch, torch.int32),
                view(fl.value, nch, torch.uint8))

    def __del__(self):
        h, self._h = getattr(self, "_h", None), None
        if h and _lib is not None:
            _lib.gnn_plan_destroy(h)


GNN_F32, GNN_BF16 = 0, 1


def _dtype_code(d):
    if d in (None, 0, "f32", "fp32", "float32", torch.float32):
        return GNN_F32
    if d in (1, "bf16", "bfloat16", torch.bfloat16):
        return GNN_BF16
    raise ValueError(f"unsupported feature dtype {d!r}")


def _opts(alpha=0, warps_per_block=0, force_chunk=0, force_vw=0, feature_dtype=0,
          deterministic=False, no_locality=False, num_sms=0, active_blocks_per_sm=0,
          l2_bytes=0):
    return PlanOpts(alpha, warps_per_block, force_chunk, force_vw, int(bool(deterministic)),
                    _dtype_code(feature_dtype), int(bool(no_locality)), num_sms,
                    active_blocks_per_sm, l2_bytes)


def plan(graph: DeviceGraph, K: int, alpha: int = 0, warps_per_block: int = 0,
         force_chunk: int = 0, force_vw: int = 0, feature_dtype=GNN_F32,
         deterministic: bool = False, no_locality: bool = False, num_sms: int = 0,
         active_blocks_per_sm: int = 0, l2_bytes: int = 0, stream=None) -> Plan:
    """gnn_plan_create: DTP/HVMA chunking + the GPU plan kernel (no host sync).
    feature_dtype: fp32 (default) or bf16 feature matrices.
    deterministic: split rows summed in chunk order without atomics (bit-reproducible).
    no_locality: plain DTP (InEq. 5), without the L2 locality cap and the chunk floor
    (DESIGN.md §3 steps 5b, 5c).  num_sms / active_blocks_per_sm / l2_bytes: device-
    parameter overrides for the plan arithmetic only (0 = the device's)."""
    L = lib()
    o = _opts(alpha, warps_per_block, force_chunk, force_vw, feature_dtype, deterministic,
              no_locality, num_sms, active_blocks_per_sm, l2_bytes)
    nbytes = L.gnn_plan_workspace_bytes(graph.M, graph.nnz, K, ctypes.byref(o))
    if nbytes == ctypes.c_size_t(-1).value:
        _check(GNN_ERR_INVALID_ARG)
    dev = graph.row_ind.device
    ws = torch.empty(max(int(nbytes), 1), dtype=torch.uint8, device=dev)
    h = ctypes.c_void_p()
    g = graph.desc()
    _check(L.gnn_plan_create(ctypes.byref(g), K, ctypes.byref(o), _ptr(ws), int(nbytes),
                             _stream(stream), ctypes.byref(h)))
    return Plan(h, ws, graph, K)


def _dense(t, name, dtypes=(torch.float32,), rows=None, cols=None, device=None):
    """Check a dense operand before its pointer reaches a kernel: CUDA, row-major 2-D,
    dtype, at least `rows` x `cols`, on `device` (the library reads / writes rows x cols
    elements at pitch stride(0); a smaller tensor would be accessed out of bounds)."""
    if (not torch.is_tensor(t) or t.dtype not in dtypes or t.dim() != 2 or t.stride(1) != 1
            or not t.is_cuda):
        raise ValueError(f"{name} must be a CUDA row-major 2-D tensor of {dtypes}")
    if (rows is not None and t.shape[0] < rows) or (cols is not None and t.shape[1] < cols):
        raise ValueError(f"{name} is {tuple(t.shape)}, needs at least ({rows}, {cols})")
    if device is not None and t.device != device:
        raise ValueError(f"{name} is on {t.device}, the graph on {device}")
    return t


def _vec_out(t, name, n, device):
    """A caller-supplied SDDMM output: contiguous fp32 CUDA vector of >= n elements."""
    if (not torch.is_tensor(t) or t.dtype != torch.float32 or not t.is_cuda
            or not t.is_contiguous() or t.numel() < n or t.device != device):
        raise ValueError(f"{name} must be a contiguous fp32 tensor of >= {n} elements on "
                         f"{device}")
    return t


_FEAT = (torch.float32, torch.bfloat16)


AGG = {"sum": 0, "mean": 1, "max": 2, "min": 3}


def spmm(p: Plan, graph: DeviceGraph, A: torch.Tensor, out: torch.Tensor | None = None,
         agg: str = "sum", accumulate: bool = False, stream=None) -> torch.Tensor:
    """gnn_spmm: O = S A (overwrites out; returns it).  agg / accumulate select
    gnn_spmm_ex: (+) in {sum, mean, max, min}; accumulate=True computes O += S A."""
    K = p.K
    dev = graph.row_ind.device
    _dense(A, "A", _FEAT, rows=graph.N if graph.nnz else 0, cols=K, device=dev)
    if out is None:
        if accumulate:
            raise ValueError("accumulate=True needs an existing out")
        out = torch.empty((graph.M, K), dtype=torch.float32, device=A.device)
    _dense(out, "out", rows=graph.M, cols=K, device=dev)
    g = graph.desc()
    if agg != "sum" or accumulate:
        _check(lib().gnn_spmm_ex(p.handle, ctypes.byref(g), _ptr(A), A.stride(0), _ptr(out),
                                 out.stride(0), AGG[agg], int(accumulate), _stream(stream)))
        return out
    fn = lib().gnn_spmm_bf16 if A.dtype == torch.bfloat16 else lib().gnn_spmm
    _check(fn(p.handle, ctypes.byref(g), _ptr(A), A.stride(0), _ptr(out), out.stride(0),
              _stream(stream)))
    return out


def spmm_extremum_backward(graph: DeviceGraph, agg: str, A: torch.Tensor, O: torch.Tensor,
                           dO: torch.Tensor, dA: torch.Tensor | None = None,
                           dval: torch.Tensor | None = None, stream=None):
    """gnn_spmm_extremum_backward: gradients of sum(dO * O) for O = spmm(..., agg=max|min)
    (the first nonzero of each row attaining the extremum takes each column's gradient).
    Accumulates into dA (N x K) / dval (nnz) when given, else returns fresh zeroed ones."""
    if agg not in ("max", "min"):
        raise ValueError("agg must be 'max' or 'min'")
    dev = graph.row_ind.device
    K = A.shape[1] if torch.is_tensor(A) and A.dim() == 2 else 0
    _dense(A, "A", rows=graph.N if graph.nnz else 0, device=dev)
    for t, n in ((O, "O"), (dO, "dO")):
        _dense(t, n, rows=graph.M, cols=K, device=dev)
    if dA is None:
        dA = torch.zeros((graph.N, K), dtype=torch.float32, device=A.device)
    _dense(dA, "dA", rows=graph.N, cols=K, device=dev)
    if dval is not None:
        _vec_out(dval, "dval", graph.nnz, dev)
    g = graph.desc()
    _check(lib().gnn_spmm_extremum_backward(ctypes.byref(g), AGG[agg], K, _ptr(A), A.stride(0),
                                            _ptr(O), O.stride(0), _ptr(dO), dO.stride(0),
                                            _ptr(dA), dA.stride(0), _ptr(dval), _stream(stream)))
    return dA, dval


class StepRunner:
    """gnn_plan_spmm_sddmm: plan + SpMM + SDDMM (A1 = A2T = X) of one device graph in a
    single native call, with a reusable plan workspace (sized for the largest graph seen)
    -- the per-step path for sampled subgraphs (BJ configs[2])."""

    def __init__(self, device="cuda"):
        self.device = device
        self.ws = torch.empty(256, dtype=torch.uint8, device=device)
        self.opts = PlanOpts()

    def __call__(self, graph: DeviceGraph, X: torch.Tensor, O: torch.Tensor | None,
                 out: torch.Tensor | None, stream=None):
        dev = graph.row_ind.device
        _dense(X, "X", rows=max(graph.N, graph.row_base + graph.M), device=dev)
        K = X.shape[1]
        if O is not None:
            _dense(O, "O", rows=graph.M, cols=K, device=dev)
        if out is not None:
            _vec_out(out, "out", graph.nnz, dev)
        L = lib()
        nbytes = L.gnn_plan_workspace_bytes(graph.M, graph.nnz, K, ctypes.byref(self.opts))
        if nbytes == ctypes.c_size_t(-1).value:
            _check(GNN_ERR_INVALID_ARG)
        if nbytes > self.ws.numel():
            self.ws = torch.empty(int(nbytes) * 2, dtype=torch.uint8, device=self.device)
        _check(L.gnn_plan_spmm_sddmm(ctypes.byref(graph.desc()), K, ctypes.byref(self.opts),
                                     _ptr(X), X.stride(0), _ptr(O),
                                     0 if O is None else O.stride(0), _ptr(out), _ptr(self.ws),
                                     self.ws.numel(), _stream(stream)))


def transpose(graph: DeviceGraph, stream=None):
    """gnn_transpose: (S^T as a DeviceGraph with row_ptr, edge_perm) on the device.
    edge_perm[j] is the edge id (index into graph's arrays) of transposed entry j."""
    L = lib()
    dev = graph.row_ind.device
    nnz = graph.nnz
    nbytes = L.gnn_transpose_workspace_bytes(nnz)
    ws = torch.empty(max(int(nbytes), 1), dtype=torch.uint8, device=dev)
    rp = torch.empty(graph.N + 1, dtype=torch.int32, device=dev)
    ri = torch.empty(nnz, dtype=torch.int32, device=dev)
    ci = torch.empty(nnz, dtype=torch.int32, device=dev)
    vt = torch.empty(nnz, dtype=torch.float32, device=dev)
    perm = torch.empty(nnz, dtype=torch.int32, device=dev)
    g = graph.desc()
    _check(L.gnn_transpose(ctypes.byref(g), _ptr(ws), int(nbytes), _ptr(rp), _ptr(ri), _ptr(ci),
                           _ptr(vt), _ptr(perm), _stream(stream)))
    gt = DeviceGraph(graph.N, graph.M, ri, ci, vt if graph.val is not None else None, rp, 0)
    return gt, perm


def gather_values(src: torch.Tensor, idx: torch.Tensor, stream=None) -> torch.Tensor:
    """gnn_gather_f32: src[idx] on the device (fp32 values, int32 indices)."""
    if (src.dtype != torch.float32 or not src.is_cuda or not src.is_contiguous()
            or idx.dtype != torch.int32 or not idx.is_contiguous() or idx.device != src.device):
        raise ValueError("gather_values: contiguous fp32 src and int32 idx on one CUDA device")
    out = torch.empty(idx.numel(), dtype=torch.float32, device=src.device)
    _check(lib().gnn_gather_f32(_ptr(src), _ptr(idx), idx.numel(), _ptr(out), _stream(stream)))
    return out


def scale_rows_inv_degree(graph: DeviceGraph, X: torch.Tensor, out: torch.Tensor | None = None,
                          stream=None) -> torch.Tensor:
    """gnn_scale_rows_inv_degree: X[r] / max(1, deg r) (the mean aggregator's backward)."""
    if graph.row_ptr is None:
        raise ValueError("scale_rows_inv_degree needs the graph's row_ptr")
    _dense(X, "X", rows=graph.M, device=graph.row_ind.device)
    if out is None:
        out = torch.empty_like(X)
    _dense(out, "out", rows=graph.M, cols=X.shape[1], device=X.device)
    _check(lib().gnn_scale_rows_inv_degree(_ptr(graph.row_ptr), graph.M, X.shape[1], _ptr(X),
                                           X.stride(0), _ptr(out), out.stride(0),
                                           _stream(stream)))
    return out


def sddmm(p: Plan, graph: DeviceGraph, A1: torch.Tensor, A2T: torch.Tensor,
          out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """gnn_sddmm: out[i] = val[i] * <A1[row_i], A2T[col_i]> (returns out)."""
    dev = graph.row_ind.device
    K = p.K
    _dense(A1, "A1", _FEAT, rows=graph.M if graph.nnz else 0, cols=K, device=dev)
    _dense(A2T, "A2T", (A1.dtype,), rows=graph.N if graph.nnz else 0, cols=K, device=dev)
    if out is None:
        out = torch.empty(graph.nnz, dtype=torch.float32, device=A1.device)
    _vec_out(out, "out", graph.nnz, dev)
    g = graph.desc()
    fn = lib().gnn_sddmm_bf16 if A1.dtype == torch.bfloat16 else lib().gnn_sddmm
    _check(fn(p.handle, ctypes.byref(g), _ptr(A1), A1.stride(0), _ptr(A2T), A2T.stride(0),
              _ptr(out), _stream(stream)))
    return out


# ---------------------------------------------------------------- helpers ---
def shard_rows(row_ptr, P: int) -> np.ndarray:
    """gnn_shard_rows on a HOST row_ptr (numpy int32)."""
    rp = np.ascontiguousarray(row_ptr, dtype=np.int32)
    b = np.empty(P + 1, np.int64)
    _check(lib().gnn_shard_rows(rp.ctypes.data, rp.shape[0] - 1, P, b.ctypes.data))
    return b


def split_col_blocks(row_ind, col_ind, val, P: int, blk: int):
    """gnn_split_col_blocks (host): stable partition of the nonzeros by column owner block
    (col // blk) -> (row_ind, col_ind, val, bounds[P+1])."""
    ri = np.ascontiguousarray(row_ind, dtype=np.int32)
    ci = np.ascontiguousarray(col_ind, dtype=np.int32)
    v = None if val is None else np.ascontiguousarray(val, dtype=np.float32)
    n = ri.shape[0]
    ro, co = np.empty(n, np.int32), np.empty(n, np.int32)
    vo = None if v is None else np.empty(n, np.float32)
    b = np.empty(P + 1, np.int64)
    _check(lib().gnn_split_col_blocks(ri.ctypes.data, ci.ctypes.data,
                                      None if v is None else v.ctypes.data, n, P, blk,
                                      ro.ctypes.data, co.ctypes.data,
                                      None if vo is None else vo.ctypes.data, b.ctypes.data))
    return ro, co, vo, b


def shard_edges(nnz: int, P: int) -> np.ndarray:
    b = np.empty(P + 1, np.int64)
    _check(lib().gnn_shard_edges(nnz, P, b.ctypes.data))
    return b


def csr_to_coo(row_ptr: torch.Tensor, row_base: int = 0, stream=None) -> torch.Tensor:
    M = row_ptr.numel() - 1
    nnz = int(row_ptr[-1].item() - row_ptr[0].item()) if M >= 0 else 0
    out = torch.empty(nnz, dtype=torch.int32, device=row_ptr.device)
    _check(lib().gnn_csr_to_coo(_ptr(row_ptr), M, row_base, _ptr(out), _stream(stream)))
    return out


def validate(graph: DeviceGraph, stream=None) -> None:
    g = graph.desc()
    _check(lib().gnn_validate(ctypes.byref(g), _stream(stream)))


# ---------------------------------------------------------------- reorder ---
def reorder_gcr(row_ptr, col_ind, max_levels=0, max_passes=0, min_gain=0.0, resolution=0.0,
                hub_rows=0):
    """gnn_reorder_gcr (host): Louvain-based GCR permutation of a square symmetric graph.
    Returns (perm, community, modularity) with perm[old] = new.  hub_rows > 0 places the
    hub_rows highest-degree nodes first (a contiguous hub block of X)."""
    rp = np.ascontiguousarray(row_ptr, dtype=np.int32)
    ci = np.ascontiguousarray(col_ind, dtype=np.int32)
    n = rp.shape[0] - 1
    perm = np.empty(n, np.int32)
    comm = np.empty(n, np.int32)
    q = ctypes.c_double(0.0)
    o = ReorderOpts(max_levels, max_passes, min_gain, resolution, hub_rows)
    _check(lib().gnn_reorder_gcr(rp.ctypes.data, ci.ctypes.data, n, ctypes.byref(o),
                                 perm.ctypes.data, comm.ctypes.data, ctypes.byref(q)))
    return perm, comm, q.value


def permute_graph(row_ptr, col_ind, val, perm):
    """gnn_permute_graph (host): S' = P S P^T -> (row_ptr, row_ind, col_ind, val)."""
    rp = np.ascontiguousarray(row_ptr, dtype=np.int32)
    ci = np.ascontiguousarray(col_ind, dtype=np.int32)
    v = None if val is None else np.ascontiguousarray(val, dtype=np.float32)
    pm = np.ascontiguousarray(perm, dtype=np.int32)
    n = rp.shape[0] - 1
    nnz = int(rp[-1]) - int(rp[0])
    orp = np.empty(n + 1, np.int32)
    ori = np.empty(nnz, np.int32)
    oci = np.empty(nnz, np.int32)
    ov = None if v is None else np.empty(nnz, np.float32)
    _check(lib().gnn_permute_graph(rp.ctypes.data, ci.ctypes.data,
                                   None if v is None else v.ctypes.data, n, pm.ctypes.data,
                                   orp.ctypes.data, ori.ctypes.data, oci.ctypes.data,
                                   None if ov is None else ov.ctypes.data))
    return orp, ori, oci, ov


def permute_rows(X: torch.Tensor, perm: torch.Tensor, out: torch.Tensor | None = None,
                 stream=None) -> torch.Tensor:
    """gnn_permute_rows (device): out[perm[i]] = X[i]."""
    _dense(X, "X")
    if out is None:
        out = torch.empty_like(X)
    _dense(out, "out", rows=X.shape[0], cols=X.shape[1], device=X.device)
    perm = perm.to(device=X.device, dtype=torch.int32).contiguous()
    if perm.numel() != X.shape[0]:
        raise ValueError("permute_rows: perm must have one entry per row of X")
    _check(lib().gnn_permute_rows(_ptr(X), X.stride(0), X.shape[0], X.shape[1], _ptr(perm),
                                  _ptr(out), out.stride(0), _stream(stream)))
    return out


def probe_gather(X: torch.Tensor, idx: torch.Tensor, sink: torch.Tensor | None = None,
                 stream=None, chunk: int = 0) -> None:
    """gnn_probe_gather: pure row gather X[idx] (measurement utility); chunk > 0 selects
    gnn_probe_gather_chunked (the kernels' traversal: one lane group per chunk)."""
    if sink is None:
        sink = torch.zeros(1, device=X.device)
    _dense(X, "X", rows=1)
    if idx.dtype != torch.int32 or not idx.is_contiguous() or idx.device != X.device:
        raise ValueError("idx must be a contiguous int32 tensor on X's device")
    if chunk:
        _check(lib().gnn_probe_gather_chunked(_ptr(X), X.stride(0), _ptr(idx), idx.numel(),
                                              X.shape[1], chunk, _ptr(sink), _stream(stream)))
        return
    _check(lib().gnn_probe_gather(_ptr(X), X.stride(0), _ptr(idx), idx.numel(), X.shape[1],
                                  _ptr(sink), _stream(stream)))


class HostRunner:
    """gnn_run_host: the end-to-end call on HOST buffers.  Holds the device workspace
    (sized for the largest K, and for run_multi over Ks if given) and the host graph
    descriptor; run() / run_multi() enqueue H2D copies, plans, SpMM, SDDMM and D2H copies
    ordered on the current stream (synchronise before reading)."""

    def __init__(self, M, N, row_ind, col_ind, val, Kmax, device="cuda", Ks=None, row_base=0,
                 row_ptr=None, **opts):
        """M rows [row_base, row_base + M) of an N-node graph (a row shard when M < N).
        row_ptr (the shard's M + 1 CSR offsets): upload those instead of RowInd."""
        self._keep = [np.ascontiguousarray(row_ind, np.int32),
                      np.ascontiguousarray(col_ind, np.int32),
                      None if val is None else np.ascontiguousarray(val, np.float32),
                      None if row_ptr is None else np.ascontiguousarray(row_ptr, np.int32)]
        if row_ptr is not None and self._keep[3].shape[0] != int(M) + 1:
            raise ValueError("row_ptr must have M + 1 entries")
        self.M, self.N, self.nnz = int(M), int(N), int(row_ind.shape[0] if hasattr(row_ind, "shape") else len(row_ind))
        self.row_base = int(row_base)
        self.opts = _opts(**opts)
        nbytes = lib().gnn_run_host_workspace_bytes(self.M, self.N, self.nnz, Kmax,
                                                    ctypes.byref(self.opts))
        if nbytes == ctypes.c_size_t(-1).value:
            _check(GNN_ERR_INVALID_ARG)
        if Ks is not None:
            karr = (ctypes.c_int32 * len(Ks))(*Ks)
            mb = lib().gnn_run_host_multi_workspace_bytes(self.M, self.N, self.nnz, len(Ks),
                                                          karr, ctypes.byref(self.opts))
            if mb == ctypes.c_size_t(-1).value:
                _check(GNN_ERR_INVALID_ARG)
            nbytes = max(int(nbytes), int(mb))
        self.ws = torch.empty(max(int(nbytes), 1), dtype=torch.uint8, device=device)
        self.ws_bytes = int(nbytes)
        self.desc = _Graph(self.M, self.N, self.nnz,
                           None if self._keep[3] is None else self._keep[3].ctypes.data,
                           self._keep[0].ctypes.data, self._keep[1].ctypes.data,
                           None if self._keep[2] is None else self._keep[2].ctypes.data, self.row_base)

    def pin(self):
        """Re-point the graph at pinned copies (asynchronous H2D)."""
        pinned = [None if a is None else torch.from_numpy(a).pin_memory() for a in self._keep]
        self._pinned = pinned
        self.desc = _Graph(self.M, self.N, self.nnz,
                           None if pinned[3] is None else pinned[3].data_ptr(),
                           pinned[0].data_ptr(), pinned[1].data_ptr(),
                           None if pinned[2] is None else pinned[2].data_ptr(), self.row_base)
        return self

    def _check_host(self, X_host, K, O_host, out_host):
        for t, n in ((X_host, self.N * K), (O_host, self.M * K), (out_host, self.nnz)):
            if t is not None and (t.is_cuda or not t.is_contiguous() or t.dtype != torch.float32
                                  or t.numel() < n):
                raise ValueError("host buffers must be contiguous fp32 CPU tensors of "
                                 "N*K (X), M*K (O) and nnz (out) elements")

    def run(self, X_host: torch.Tensor, K: int, O_host=None, out_host=None, upload_graph=True,
            stream=None):
        self._check_host(X_host, K, O_host, out_host)
        _check(lib().gnn_run_host(ctypes.byref(self.desc), int(upload_graph), _ptr(X_host), K,
                                  _ptr(O_host), _ptr(out_host), ctypes.byref(self.opts),
                                  _ptr(self.ws), self.ws_bytes, _stream(stream)))

    def run_multi(self, X_hosts, Ks, O_hosts=None, out_hosts=None, upload_graph=True,
                  stream=None):
        """gnn_run_host_multi: several feature widths on one graph in one pipelined call
        (later X uploads and every download overlap the kernels of earlier widths)."""
        n = len(Ks)
        O_hosts = O_hosts or [None] * n
        out_hosts = out_hosts or [None] * n
        if not (len(X_hosts) == len(O_hosts) == len(out_hosts) == n):
            raise ValueError("run_multi: one X / O / out entry per width")
        for X_host, K, O_host, out_host in zip(X_hosts, Ks, O_hosts, out_hosts):
            self._check_host(X_host, K, O_host, out_host)
        vp = ctypes.c_void_p
        karr = (ctypes.c_int32 * n)(*Ks)
        xa = (vp * n)(*[_ptr(t) for t in X_hosts])
        oa = (vp * n)(*[_ptr(t) for t in O_hosts])
        ea = (vp * n)(*[_ptr(t) for t in out_hosts])
        _check(lib().gnn_run_host_multi(ctypes.byref(self.desc), int(upload_graph), n, karr, xa,
                                        oa, ea, ctypes.byref(self.opts), _ptr(self.ws),
                                        self.ws_bytes, _stream(stream)))
