"""Workload recipes C1-C5 (BASELINE.json ``configs``; recipe in DESIGN.md).

Every graph is symmetric, self-looped, deduplicated, randomly
relabelled, sorted by (row, col): hybrid CSR/COO.  Shapes follow the paper's
datasets (Table II): Reddit 232,965 / 114,848,857 and ogbn-products
2,449,029 / 126,167,053 (counts include the self-loops).
"""
from __future__ import annotations

import numpy as np

from . import powerlaw_graph, features

CONFIGS = {
    # BJ configs[0]: tiny power-law graph N=1000, nnz=10000, K=32, vs CPU oracle
    "C1": dict(n=1000, nnz=10_000, gamma=2.5, max_deg=200, n_comm=4, mu=0.3,
               val_mode="uniform", seed=1, K=[32]),
    # BJ configs[1]: Cora/PubMed-shaped GCN graph N~20k nnz~100k, K=64, full graph
    "C2": dict(n=20_000, nnz=100_000, gamma=2.8, max_deg=0, n_comm=20, mu=0.3,
               val_mode="gcn", seed=2, K=[64]),
    # BJ configs[3]: Reddit-shaped N=232,965 nnz=114,848,857, K=32..256, 1/2/4/8 GPUs
    "C4": dict(n=232_965, nnz=114_848_857, gamma=2.2, max_deg=20_000, n_comm=50, mu=0.3,
               val_mode="gcn", seed=4, K=[32, 64, 128, 256]),
    # BJ configs[4]: ogbn-products-shaped N=2,449,029 nnz=126,167,053, K=256
    "C5": dict(n=2_449_029, nnz=126_167_053, gamma=2.3, max_deg=17_000, n_comm=500, mu=0.3,
               val_mode="gcn", seed=5, K=[256]),
}

FEATURE_SEED = {"C1": 1001, "C2": 1002, "C3": 1003, "C4": 1004, "C5": 1005}


def make_graph(name: str, scale: float = 1.0):
    """Generate config `name`; scale < 1 shrinks n and nnz proportionally (tests)."""
    c = CONFIGS[name]
    n = max(2, int(round(c["n"] * scale)))
    nnz = max(n, int(round(c["nnz"] * scale)))
    md = c["max_deg"] * scale if c["max_deg"] else 0
    return powerlaw_graph(n, nnz, gamma=c["gamma"], max_deg=md, n_comm=max(1, int(c["n_comm"])),
                          mu=c["mu"], val_mode=c["val_mode"], seed=c["seed"])


def c3_params(t: int):
    """BJ configs[2]: GraphSAINT-style sampled subgraph t (new graph every step):
    N_t ~ U[8k, 50k], average degree ~ U[15, 30] (the paper's sampled graphs have
    average degree 21-25), power law gamma 2.3, GCN values."""
    r = np.random.default_rng(3_000 + t)
    n = int(r.integers(8_000, 50_001))
    deg = float(r.uniform(15, 30))
    return dict(n=n, nnz=int(n * deg), gamma=2.3, max_deg=0, n_comm=max(1, n // 1000),
                mu=0.3, val_mode="gcn", seed=300 + t)


def make_c3(t: int):
    p = c3_params(t)
    return powerlaw_graph(p["n"], p["nnz"], gamma=p["gamma"], max_deg=p["max_deg"],
                          n_comm=p["n_comm"], mu=p["mu"], val_mode=p["val_mode"], seed=p["seed"])


def make_features(name: str, rows: int, K: int, which: int = 0, row0: int = 0):
    return features(FEATURE_SEED.get(name, 999) * 16 + which, rows, K, row0=row0)
