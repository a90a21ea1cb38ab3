"""Seeded synthetic-input generators (the only module both sides share).

Holds none of the method's arithmetic: it produces hybrid CSR/COO graphs
(Fig. 2d) and dense fp32 feature matrices from a seed, via the
C library ``gen/libgnngen.so`` (counter-based RNG, thread-count independent).

The workload recipes C1-C5 (BASELINE.json ``configs``) live in ``gen.configs``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libgnngen.so")
_lib = None


class _Params(ctypes.Structure):
    _fields_ = [
        ("n", ctypes.c_int64),
        ("target_nnz", ctypes.c_int64),
        ("gamma", ctypes.c_double),
        ("max_deg", ctypes.c_double),
        ("n_comm", ctypes.c_int32),
        ("mu", ctypes.c_double),
        ("relabel", ctypes.c_int32),
        ("val_mode", ctypes.c_int32),
        ("seed", ctypes.c_uint64),
    ]


def _load():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        root = os.path.dirname(_HERE)
        subprocess.check_call(["make", "-C", root, "gen/libgnngen.so"],
                              stdout=subprocess.DEVNULL)
    lib = ctypes.CDLL(_LIB_PATH)
    P = ctypes.POINTER
    lib.gen_graph_nnz.argtypes = [P(_Params)]
    lib.gen_graph_nnz.restype = ctypes.c_int64
    lib.gen_graph.argtypes = [P(_Params), ctypes.c_void_p, ctypes.c_void_p,
                              ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                              ctypes.c_int64, P(ctypes.c_int64)]
    lib.gen_graph.restype = ctypes.c_int
    lib.gen_features.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_int64,
                                 ctypes.c_int64, ctypes.c_int64, ctypes.c_void_p]
    lib.gen_features.restype = None
    lib.gen_values_uniform.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_void_p]
    lib.gen_values_uniform.restype = None
    _lib = lib
    return lib


@dataclass
class Graph:
    """Hybrid CSR/COO adjacency: row_ptr[M+1] plus the fully decoded
    row_ind[nnz], col_ind[nnz], val[nnz]; rows non-decreasing, cols sorted per row."""
    M: int
    N: int
    row_ptr: np.ndarray
    row_ind: np.ndarray
    col_ind: np.ndarray
    val: np.ndarray
    comm: np.ndarray | None = None

    @property
    def nnz(self) -> int:
        return int(self.row_ind.shape[0])

    def degree_stats(self) -> dict:
        d = np.diff(self.row_ptr.astype(np.int64))
        if d.size == 0:
            return {"mean": 0.0, "std": 0.0, "max": 0}
        return {"mean": float(d.mean()), "std": float(d.std()), "max": int(d.max())}


def powerlaw_graph(n: int, nnz: int, gamma: float = 2.3, max_deg: float = 0.0,
                   n_comm: int = 1, mu: float = 0.3, relabel: bool = True,
                   val_mode: str = "gcn", seed: int = 0) -> Graph:
    """Symmetric self-looped power-law graph with planted communities; nnz is
    n + 2*floor((nnz-n)/2) exactly.  val_mode: 'uniform' U(0,1], 'gcn'
    1/sqrt(deg_r deg_c), 'ones'."""
    lib = _load()
    vm = {"uniform": 0, "gcn": 1, "ones": 2}[val_mode]
    p = _Params(n, nnz, gamma, max_deg, n_comm, mu, int(relabel), vm,
                ctypes.c_uint64(seed & 0xFFFFFFFFFFFFFFFF).value)
    cap = lib.gen_graph_nnz(ctypes.byref(p))
    row_ptr = np.empty(n + 1, np.int32)
    row_ind = np.empty(cap, np.int32)
    col_ind = np.empty(cap, np.int32)
    val = np.empty(cap, np.float32)
    comm = np.empty(n, np.int32)
    out = ctypes.c_int64(0)
    rc = lib.gen_graph(ctypes.byref(p), row_ptr.ctypes.data, row_ind.ctypes.data,
                       col_ind.ctypes.data, val.ctypes.data, comm.ctypes.data, cap,
                       ctypes.byref(out))
    if rc != 0:
        raise RuntimeError(f"gen_graph failed (rc={rc}) for n={n} nnz={nnz}")
    m = out.value
    return Graph(n, n, row_ptr, row_ind[:m], col_ind[:m], val[:m], comm)


def features(seed: int, rows: int, K: int, row0: int = 0, ld: int | None = None,
             out: np.ndarray | None = None) -> np.ndarray:
    """X[i][k] = U(-1,1) from counter (seed, (row0+i)*K + k); odd multiples of 2^-24,
    so never zero or subnormal.  Row-major rows x ld (ld >= K)."""
    lib = _load()
    ld = K if ld is None else ld
    if out is None:
        out = np.zeros((rows, ld), np.float32)
    assert out.dtype == np.float32 and out.flags.c_contiguous and out.shape[1] == ld
    lib.gen_features(ctypes.c_uint64(seed).value, row0, rows, K, ld, out.ctypes.data)
    return out


def uniform_values(seed: int, nnz: int) -> np.ndarray:
    lib = _load()
    v = np.empty(nnz, np.float32)
    lib.gen_values_uniform(ctypes.c_uint64(seed).value, nnz, v.ctypes.data)
    return v


def from_coo(M: int, N: int, rows, cols, vals=None) -> Graph:
    """Build a Graph from explicit (row, col[, val]) triples, sorted by row
    (stable: column order within a row is kept; duplicates are kept)."""
    rows = np.asarray(rows, np.int64)
    cols = np.asarray(cols, np.int64)
    vals = np.ones(rows.shape[0], np.float32) if vals is None else np.asarray(vals, np.float32)
    order = np.argsort(rows, kind="stable")
    rows, cols, vals = rows[order], cols[order], vals[order]
    row_ptr = np.zeros(M + 1, np.int64)
    np.add.at(row_ptr, rows + 1, 1)
    row_ptr = np.cumsum(row_ptr).astype(np.int32)
    return Graph(M, N, row_ptr, rows.astype(np.int32), cols.astype(np.int32),
                 vals.astype(np.float32))
