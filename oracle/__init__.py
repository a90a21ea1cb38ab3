"""CPU oracle -- TEST INFRASTRUCTURE ONLY.

Plain fp64 C implementation (``oracle/oracle.c``) of what the hot path computes:
Algorithm 1 SpMM, Algorithm 2 SDDMM, the DTP/HVMA
plan (restated in DESIGN.md "Plan rule"), nnz-balanced shards and
CSR->COO decoding.  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this module.  It shares no
code with ``paper_conf_ipps_fanwc23_b200`` (the CUDA path) and neither imports the
other.  Pins: tests/test_oracle.py (see oracle.h header for the list).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None


class _PlanInfo(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in (
        "chunk", "vw_feat", "vw_sparse", "lanes", "vecs", "slices", "groups",
        "warps_per_block", "active_blocks_per_sm", "num_sms", "alpha", "K",
        "feature_dtype", "chunk_dtp")] + [
        ("nnz", ctypes.c_int64), ("num_chunks", ctypes.c_int64),
        ("num_blocks", ctypes.c_int64), ("M", ctypes.c_int64), ("l2_bytes", ctypes.c_int64)]


def _load():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        root = os.path.dirname(_HERE)
        subprocess.check_call(["make", "-C", root, "oracle/liboracle.so"],
                              stdout=subprocess.DEVNULL)
    lib = ctypes.CDLL(_LIB_PATH)
    vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
    lib.oracle_spmm.argtypes = [i64, i64, vp, vp, vp, i64, vp, i64, i64, i64, vp, vp]
    lib.oracle_sddmm.argtypes = [i64, i64, vp, vp, vp, i64, vp, i64, vp, i64, vp, vp]
    lib.oracle_spmm_agg.argtypes = [i64, i64, vp, vp, vp, i64, vp, i64, i64, i64, i32, vp, vp]
    lib.oracle_spmm_extremum_backward.argtypes = [i64, i64, vp, vp, vp, i64, vp, i64, i64, i64,
                                                  i64, i32, vp, vp, vp]
    lib.oracle_plan.argtypes = [i64, vp, i32, i32, i32, i32, i32, i32, i32, i32, i64, i64,
                                ctypes.POINTER(_PlanInfo), vp, vp, vp]
    lib.oracle_shard_rows.argtypes = [vp, i64, i32, vp]
    lib.oracle_shard_edges.argtypes = [i64, i32, vp]
    lib.oracle_csr_to_coo.argtypes = [vp, i64, vp]
    lib.oracle_modularity.argtypes = [vp, vp, i64, vp, i32]
    lib.oracle_modularity.restype = ctypes.c_double
    lib.oracle_threads.argtypes = [ctypes.c_int]
    lib.oracle_threads.restype = ctypes.c_int
    for f in ("oracle_spmm", "oracle_spmm_agg", "oracle_sddmm", "oracle_plan", "oracle_shard_rows",
              "oracle_shard_edges", "oracle_csr_to_coo"):
        getattr(lib, f).restype = ctypes.c_int
    _lib = lib
    return lib


def threads(n: int = 0) -> int:
    """Set the oracle's OpenMP thread count (n > 0); returns the count in effect."""
    return int(_load().oracle_threads(n))


def _i32(a):
    return np.ascontiguousarray(a, dtype=np.int32)


def _f32_2d(a):
    a = np.asarray(a)
    assert a.dtype == np.float32 and a.ndim == 2 and a.strides[1] == 4, \
        "dense operands must be row-major fp32"
    return a


def _ptr(a):
    return None if a is None else a.ctypes.data


def spmm(row_ind, col_ind, val, A, M=None, i0=0, i1=None, r0=0, nrows=None):
    """Algorithm 1 over nnz [i0, i1): returns (O, T) fp64 (nrows x K), row r at r-r0.
    T[r][k] = sum |v A[c][k]| (the error-bound scale)."""
    lib = _load()
    row_ind, col_ind = _i32(row_ind), _i32(col_ind)
    val = None if val is None else np.ascontiguousarray(val, np.float32)
    A = _f32_2d(A)
    i1 = row_ind.shape[0] if i1 is None else i1
    if nrows is None:
        nrows = (M if M is not None else (int(row_ind.max()) + 1 if row_ind.size else 0)) - r0
    K = A.shape[1]
    O = np.empty((nrows, K), np.float64)
    T = np.empty((nrows, K), np.float64)
    rc = lib.oracle_spmm(i0, i1, _ptr(row_ind), _ptr(col_ind), _ptr(val), K, _ptr(A),
                         A.strides[0] // 4, r0, nrows, _ptr(O), _ptr(T))
    if rc != 0:
        raise ValueError("oracle_spmm: invalid arguments")
    return O, T


AGG = {"sum": 0, "mean": 1, "max": 2, "min": 3}


def spmm_agg(row_ind, col_ind, val, A, agg, M=None, i0=0, i1=None, r0=0, nrows=None):
    """Eq. 1 node-wise op with (+) = agg in {sum, mean, max, min}: returns (O, T)."""
    lib = _load()
    row_ind, col_ind = _i32(row_ind), _i32(col_ind)
    val = None if val is None else np.ascontiguousarray(val, np.float32)
    A = _f32_2d(A)
    i1 = row_ind.shape[0] if i1 is None else i1
    if nrows is None:
        nrows = (M if M is not None else (int(row_ind.max()) + 1 if row_ind.size else 0)) - r0
    K = A.shape[1]
    O = np.empty((nrows, K), np.float64)
    T = np.empty((nrows, K), np.float64)
    rc = lib.oracle_spmm_agg(i0, i1, _ptr(row_ind), _ptr(col_ind), _ptr(val), K, _ptr(A),
                             A.strides[0] // 4, r0, nrows, AGG[agg], _ptr(O), _ptr(T))
    if rc != 0:
        raise ValueError("oracle_spmm_agg: invalid arguments")
    return O, T


def spmm_extremum_backward(row_ind, col_ind, val, A, dO, agg, M=None):
    """Gradients (dA N x K, dval nnz) of sum(dO * O) for O = spmm_agg(..., agg) with
    agg in {max, min}: the first nonzero of each row attaining the fp32 extremum takes
    the gradient of each (row, column) (oracle.c, reading 26)."""
    lib = _load()
    row_ind, col_ind = _i32(row_ind), _i32(col_ind)
    val = None if val is None else np.ascontiguousarray(val, np.float32)
    A = _f32_2d(A)
    dO = np.ascontiguousarray(dO, np.float32)
    nrows = M if M is not None else (int(row_ind.max()) + 1 if row_ind.size else 0)
    N, K = A.shape
    assert dO.shape == (nrows, K)
    dA = np.empty((N, K), np.float64)
    dval = np.empty(row_ind.shape[0], np.float64)
    rc = lib.oracle_spmm_extremum_backward(0, row_ind.shape[0], _ptr(row_ind), _ptr(col_ind),
                                           _ptr(val), K, _ptr(A), A.strides[0] // 4, N, 0,
                                           nrows, AGG[agg], _ptr(dO), _ptr(dA), _ptr(dval))
    if rc != 0:
        raise ValueError("oracle_spmm_extremum_backward: invalid arguments")
    return dA, dval


def spmm_rows(g, A, rows):
    """Oracle rows for a sample of output rows (full-size parity): returns (O, T)
    with one row per entry of ``rows``; each row is Algorithm 1 over that row's nnz."""
    K = A.shape[1]
    O = np.empty((len(rows), K), np.float64)
    T = np.empty((len(rows), K), np.float64)
    for j, r in enumerate(rows):
        i0, i1 = int(g.row_ptr[r]), int(g.row_ptr[r + 1])
        O[j:j + 1], T[j:j + 1] = spmm(g.row_ind, g.col_ind, g.val, A, i0=i0, i1=i1,
                                      r0=int(r), nrows=1)
    return O, T


def sddmm_edges(g, A1, A2T, edges):
    """Oracle outputs for a sample of edge ids (full-size parity): (out, T), each edge
    Algorithm 2 over that one nonzero."""
    out = np.empty(len(edges), np.float64)
    T = np.empty(len(edges), np.float64)
    for j, e in enumerate(edges):
        a, b = sddmm(g.row_ind, g.col_ind, g.val, A1, A2T, i0=int(e), i1=int(e) + 1)
        out[j], T[j] = a[0], b[0]
    return out, T


def sddmm(row_ind, col_ind, val, A1, A2T, i0=0, i1=None):
    """Algorithm 2 over nnz [i0, i1): returns (out, T) fp64 of length i1-i0."""
    lib = _load()
    row_ind, col_ind = _i32(row_ind), _i32(col_ind)
    val = None if val is None else np.ascontiguousarray(val, np.float32)
    A1, A2T = _f32_2d(A1), _f32_2d(A2T)
    assert A1.shape[1] == A2T.shape[1]
    i1 = row_ind.shape[0] if i1 is None else i1
    K = A1.shape[1]
    out = np.empty(i1 - i0, np.float64)
    T = np.empty(i1 - i0, np.float64)
    rc = lib.oracle_sddmm(i0, i1, _ptr(row_ind), _ptr(col_ind), _ptr(val), K, _ptr(A1),
                          A1.strides[0] // 4, _ptr(A2T), A2T.strides[0] // 4,
                          _ptr(out), _ptr(T))
    if rc != 0:
        raise ValueError("oracle_sddmm: invalid arguments")
    return out, T


@dataclass
class Plan:
    info: dict
    row_first: np.ndarray
    row_last: np.ndarray
    flags: np.ndarray


def plan(row_ind, K, num_sms, active_blocks_per_sm, alpha=2, warps_per_block=8,
         force_chunk=0, force_vw=0, feature_dtype=0, M=0, l2_bytes=0) -> Plan:
    """DTP/HVMA plan; device parameters are inputs.  M (graph
    rows) and l2_bytes (device L2) feed the locality cap, step 5b; l2_bytes = 0 is the
    plain DTP rule."""
    lib = _load()
    row_ind = _i32(row_ind)
    nnz = row_ind.shape[0]
    info = _PlanInfo()
    # first call sizes the arrays (chunk depends on the rule)
    rc = lib.oracle_plan(nnz, _ptr(row_ind), K, alpha, warps_per_block, force_chunk,
                         force_vw, feature_dtype, num_sms, active_blocks_per_sm, M, l2_bytes,
                         ctypes.byref(info), None, None, None)
    if rc != 0:
        raise ValueError("oracle_plan: invalid arguments")
    nch = info.num_chunks
    rf = np.empty(nch, np.int32)
    rl = np.empty(nch, np.int32)
    fl = np.empty(nch, np.uint8)
    lib.oracle_plan(nnz, _ptr(row_ind), K, alpha, warps_per_block, force_chunk,
                    force_vw, feature_dtype, num_sms, active_blocks_per_sm, M, l2_bytes,
                    ctypes.byref(info), _ptr(rf), _ptr(rl), _ptr(fl))
    d = {name: getattr(info, name) for name, _ in _PlanInfo._fields_}
    return Plan(d, rf, rl, fl)


def shard_rows(row_ptr, P):
    lib = _load()
    row_ptr = _i32(row_ptr)
    b = np.empty(P + 1, np.int64)
    if lib.oracle_shard_rows(_ptr(row_ptr), row_ptr.shape[0] - 1, P, _ptr(b)) != 0:
        raise ValueError("oracle_shard_rows: invalid arguments")
    return b


def shard_edges(nnz, P):
    lib = _load()
    b = np.empty(P + 1, np.int64)
    if lib.oracle_shard_edges(nnz, P, _ptr(b)) != 0:
        raise ValueError("oracle_shard_edges: invalid arguments")
    return b


def csr_to_coo(row_ptr):
    lib = _load()
    row_ptr = _i32(row_ptr)
    M = row_ptr.shape[0] - 1
    out = np.empty(int(row_ptr[M]) - int(row_ptr[0]), np.int32)
    if lib.oracle_csr_to_coo(_ptr(row_ptr), M, _ptr(out)) != 0:
        raise ValueError("oracle_csr_to_coo: invalid arguments")
    return out


def modularity(row_ptr, col_ind, comm, skip_self=True):
    """Modularity of partition `comm` of the symmetric unit-weight CSR graph."""
    lib = _load()
    rp, ci, cm = _i32(row_ptr), _i32(col_ind), _i32(comm)
    return lib.oracle_modularity(_ptr(rp), _ptr(ci), rp.shape[0] - 1, _ptr(cm), int(skip_self))
