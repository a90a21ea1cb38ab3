"""GCR reorder: host Louvain + permutation (CPU; no GPU needed).

The community assignment itself is parity-unpinned (Louvain is a heuristic and the
paper prints no example); validity and quality are pinned: perm is a bijection, the
reported modularity equals the oracle's modularity of the returned partition, the
partition is at least as good as the planted one, the permuted graph equals the plain
definition S' = P S P^T, and the oracle's modularity is pinned to networkx."""
import networkx as nx
import numpy as np
import pytest

import gen
import oracle
import paper_conf_ipps_fanwc23_b200 as gs


def nx_graph(g):
    G = nx.Graph()
    G.add_nodes_from(range(g.M))
    G.add_edges_from((int(r), int(c)) for r, c in zip(g.row_ind, g.col_ind) if r != c)
    return G


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_oracle_modularity_pinned_to_networkx_and_bruteforce(seed):
    g = gen.powerlaw_graph(300, 3000, gamma=2.4, n_comm=4, seed=seed)
    rng = np.random.default_rng(seed)
    comm = rng.integers(0, 5, g.M).astype(np.int32)
    q = oracle.modularity(g.row_ptr, g.col_ind, comm)
    G = nx_graph(g)
    parts = [set(np.flatnonzero(comm == c).tolist()) for c in range(5)]
    parts = [p for p in parts if p]
    assert abs(q - nx.community.modularity(G, parts)) < 1e-12
    # brute-force double sum of the definition
    A = np.zeros((g.M, g.M))
    mask = g.row_ind != g.col_ind
    A[g.row_ind[mask], g.col_ind[mask]] = 1.0
    k = A.sum(1)
    m2 = k.sum()
    same = comm[:, None] == comm[None, :]
    qb = ((A - np.outer(k, k) / m2) * same).sum() / m2
    assert abs(q - qb) < 1e-12


@pytest.mark.parametrize("n,nnz,nc,seed", [(2000, 40000, 8, 1), (5000, 100000, 20, 2),
                                          (20000, 400000, 20, 5)])
def test_gcr_partition_quality_and_reported_modularity(n, nnz, nc, seed):
    g = gen.powerlaw_graph(n, nnz, gamma=2.3, n_comm=nc, mu=0.3, seed=seed)
    perm, comm, q = gs.reorder_gcr(g.row_ptr, g.col_ind)
    assert np.array_equal(np.sort(perm), np.arange(n))
    assert abs(q - oracle.modularity(g.row_ptr, g.col_ind, comm)) < 1e-9
    q_planted = oracle.modularity(g.row_ptr, g.col_ind, g.comm)
    assert q >= 0.98 * q_planted  # Louvain is greedy: within 2% of the planted optimum
    # communities are contiguous in the new order
    newcomm = np.empty(n, np.int32)
    newcomm[perm] = comm
    changes = np.count_nonzero(np.diff(newcomm))
    assert changes == len(np.unique(comm)) - 1


def test_gcr_deterministic_and_close_to_networkx_louvain():
    g = gen.powerlaw_graph(3000, 60000, gamma=2.3, n_comm=10, mu=0.3, seed=9)
    a = gs.reorder_gcr(g.row_ptr, g.col_ind)
    b = gs.reorder_gcr(g.row_ptr, g.col_ind)
    assert np.array_equal(a[0], b[0]) and a[2] == b[2]
    parts = nx.community.louvain_communities(nx_graph(g), seed=0)
    q_nx = nx.community.modularity(nx_graph(g), parts)
    assert a[2] >= q_nx - 0.02


def test_permute_graph_matches_definition():
    g = gen.powerlaw_graph(1500, 30000, seed=11)
    perm = np.random.default_rng(0).permutation(g.M).astype(np.int32)
    rp, ri, ci, v = gs.permute_graph(g.row_ptr, g.col_ind, g.val, perm)
    nr, nc_ = perm[g.row_ind], perm[g.col_ind]
    order = np.lexsort((nc_, nr))
    assert np.array_equal(ri, nr[order]) and np.array_equal(ci, nc_[order])
    assert np.array_equal(v, g.val[order])
    assert np.array_equal(rp, np.r_[0, np.cumsum(np.bincount(nr, minlength=g.M))])
    # degree multiset preserved
    assert np.array_equal(np.sort(np.diff(rp)), np.sort(np.diff(g.row_ptr)))


def test_permute_graph_rejects_non_bijection():
    g = gen.powerlaw_graph(100, 1000, seed=12)
    bad = np.zeros(100, np.int32)
    with pytest.raises(gs.GnnError):
        gs.permute_graph(g.row_ptr, g.col_ind, g.val, bad)


@pytest.mark.parametrize("H", [1, 50, 400])
def test_hub_block_first(H):
    """hub_rows = H: the H highest-degree nodes (ties: smaller id) take new ids [0, H); hubs
    and non-hubs each keep the relative order of the plain GCR permutation; bijection."""
    g = gen.powerlaw_graph(3000, 60000, gamma=2.1, n_comm=6, seed=21)
    p0, c0, q0 = gs.reorder_gcr(g.row_ptr, g.col_ind)
    p1, c1, q1 = gs.reorder_gcr(g.row_ptr, g.col_ind, hub_rows=H)
    assert sorted(p1) == list(range(g.N))
    assert np.array_equal(c0, c1) and q0 == q1
    deg = np.diff(g.row_ptr.astype(np.int64))
    top = sorted(range(g.N), key=lambda v: (-deg[v], v))[:H]
    assert set(np.flatnonzero(p1 < H)) == set(top)
    hub = p1 < H
    for mask in (hub, ~hub):
        nodes = np.flatnonzero(mask)
        assert np.array_equal(np.argsort(p1[nodes]), np.argsort(p0[nodes]))
