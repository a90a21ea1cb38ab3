"""GPU parity: the CUDA path (through the C ABI) against the fp64 CPU oracle.

Bars (BASELINE.json north_star): plan arrays/info bit-exact; fp32 outputs within
|err| <= 1e-5 * sum|terms| elementwise (tests/helpers.assert_within); exact where
the mathematics makes the result exact (one-term sums, integer sums, symmetric pairs,
sharded SDDMM vs unsharded).
"""
import numpy as np
import pytest
import torch

import gen
import oracle
from gen import configs
import paper_conf_ipps_fanwc23_b200 as gs

from helpers import assert_within, oracle_plan_checked, upload

pytestmark = pytest.mark.gpu

DEV = "cuda"


def _x(seed, rows, K, ld=None):
    X = gen.features(seed, rows, K, ld=ld)
    return X


def check_plan(p, g, K, **kw):
    """Plan info + arrays bit-exact with the oracle, which gets the device parameters
    from torch and the cuobjdump-derived occupancy (helpers.oracle_plan_checked)."""
    return oracle_plan_checked(p, g, K, **kw)


def run_full(g, K, seed=7, check_sddmm=True, with_val=True, ld_pad=0, **kw):
    """Plan + SpMM + SDDMM on the whole graph, compared with the oracle everywhere."""
    dg = upload(g, with_val=with_val)
    p = gs.plan(dg, K, **kw)
    info = check_plan(p, g, K, **kw)
    ld = K + ld_pad
    A = _x(seed, g.N, K, ld=ld)
    At = torch.from_numpy(A).to(DEV)[:, :K] if ld_pad else torch.from_numpy(A).to(DEV)
    O = torch.full((g.M, ld), float("nan"), device=DEV)[:, :K] if ld_pad else \
        torch.full((g.M, K), float("nan"), device=DEV)
    gs.spmm(p, dg, At, out=O)
    torch.cuda.synchronize()
    val = g.val if with_val else None
    ref, T = oracle.spmm(g.row_ind, g.col_ind, val, np.ascontiguousarray(A[:, :K]), M=g.M)
    worst = assert_within(O.cpu().numpy(), ref, T, what=f"spmm K={K}")
    if check_sddmm:
        A1 = _x(seed + 1, g.M, K)
        out = gs.sddmm(p, dg, torch.from_numpy(A1).to(DEV), At)
        torch.cuda.synchronize()
        r2, T2 = oracle.sddmm(g.row_ind, g.col_ind, val, A1, np.ascontiguousarray(A[:, :K]))
        assert_within(out.cpu().numpy(), r2, T2, what=f"sddmm K={K}")
    return info, worst


# ------------------------------------------------------- BJ small configs ---
def test_c1_tiny_powerlaw_k32():
    g = configs.make_graph("C1")
    info, _ = run_full(g, 32)
    assert info["chunk_dtp"] == 8  # Eq. 5 infeasible on 148 SMs -> most parallel candidate
    assert info["chunk"] == 64     # ... raised by the step-5c chunk floor


def test_c2_cora_shaped_k64():
    g = configs.make_graph("C2")
    run_full(g, 64)


@pytest.mark.parametrize("t", [0, 1, 2])
def test_c3_sampled_subgraph_k128(t):
    run_full(configs.make_c3(t), 128)


# ------------------------------------------------------ shapes / edge cases --
@pytest.mark.parametrize("K", [1, 2, 3, 4, 6, 8, 16, 24, 32, 33, 64, 100, 128, 256, 300, 512,
                               1000, 2048])
def test_feature_widths(K):
    g = gen.powerlaw_graph(3000, 60000, gamma=2.3, n_comm=6, seed=K)
    run_full(g, K)


@pytest.mark.parametrize("C", [1, 2, 5, 8, 32, 64, 128, 256, 512, 1000])
def test_forced_chunk_sizes(C):
    g = gen.powerlaw_graph(2000, 50000, gamma=2.1, n_comm=4, seed=100 + C)
    run_full(g, 32, force_chunk=C)
    run_full(g, 256, force_chunk=C)


@pytest.mark.parametrize("vw", [1, 2, 4, 8])
def test_forced_vector_width(vw):
    g = gen.powerlaw_graph(2000, 30000, seed=200 + vw)
    run_full(g, 64, force_vw=vw)


@pytest.mark.parametrize("wpb,alpha", [(1, 1), (8, 2), (16, 8)])
def test_block_shape_and_alpha(wpb, alpha):
    g = gen.powerlaw_graph(5000, 200000, seed=300 + wpb)
    run_full(g, 64, warps_per_block=wpb, alpha=alpha)


def test_val_none_and_padded_pitch():
    g = gen.powerlaw_graph(3000, 40000, seed=301)
    run_full(g, 64, with_val=False)
    run_full(g, 64, ld_pad=16)            # pitch 80: a multiple of VW = 8
    run_full(g, 64, ld_pad=12, force_vw=4)  # pitch 76 needs a narrower vector width


def test_pitch_incompatible_with_vector_width_is_unsupported():
    g = gen.powerlaw_graph(500, 5000, seed=302)
    dg = upload(g)
    p = gs.plan(dg, 64)
    assert p.info()["vw_feat"] == 8
    A = torch.zeros((g.N, 76), device=DEV)[:, :64]
    with pytest.raises(gs.GnnError) as e:
        gs.spmm(p, dg, A)
    assert e.value.status == gs.GNN_ERR_UNSUPPORTED


def test_empty_rows_rectangular_duplicates():
    rng = np.random.default_rng(5)
    M, N, nnz = 777, 333, 9000
    rows = rng.integers(0, M, nnz)
    rows = rows[(rows % 7) != 3]  # many empty rows, incl. runs
    rows = np.concatenate([rows, np.full(3000, 500)])  # one heavy row
    cols = rng.integers(0, N, rows.size)
    cols[:20] = cols[0]
    rows[:20] = rows[0]  # duplicates
    vals = rng.uniform(0.1, 1, rows.size).astype(np.float32)
    g = gen.from_coo(M, N, rows, cols, vals)
    for C in (0, 5, 8, 64, 512):
        run_full(g, 32, force_chunk=C)
        run_full(g, 12, force_chunk=C)


def test_leading_and_trailing_empty_rows():
    g = gen.from_coo(50, 10, [10, 10, 11, 30, 30, 30], [1, 2, 3, 4, 5, 6])
    for C in (0, 1, 2, 4):
        run_full(g, 8, force_chunk=C)


def test_single_hub_row_spans_many_chunks():
    N = 20000
    g = gen.from_coo(3, N, np.r_[np.zeros(5), np.ones(N), np.full(5, 2)],
                     np.r_[np.arange(5), np.arange(N), np.arange(5)],
                     gen.uniform_values(9, N + 10))
    for C in (0, 8, 64, 512):
        run_full(g, 128, force_chunk=C)


def test_empty_graph_overwrites_output():
    g = gen.from_coo(40, 10, [], [])
    dg = upload(g)
    p = gs.plan(dg, 16)
    assert p.info()["num_chunks"] == 0
    O = torch.full((40, 16), 7.0, device=DEV)
    gs.spmm(p, dg, torch.zeros((10, 16), device=DEV), out=O)
    out = gs.sddmm(p, dg, torch.zeros((40, 16), device=DEV), torch.zeros((10, 16), device=DEV))
    torch.cuda.synchronize()
    assert (O == 0).all() and out.numel() == 0


def test_zero_rows_graph():
    g = gen.from_coo(0, 10, [], [])
    dg = upload(g)
    p = gs.plan(dg, 8)
    gs.spmm(p, dg, torch.zeros((10, 8), device=DEV), out=torch.empty((0, 8), device=DEV))


# ------------------------------------------------------------ exact pins ---
def test_identity_returns_A_bitwise():
    N, K = 5000, 64
    g = gen.from_coo(N, N, np.arange(N), np.arange(N))
    A = torch.from_numpy(_x(1, N, K)).to(DEV)
    dg = upload(g)
    for C in (0, 1, 8, 512):
        p = gs.plan(dg, K, force_chunk=C)
        O = gs.spmm(p, dg, A)
        torch.cuda.synchronize()
        assert torch.equal(O, A)


def test_ones_features_integer_sums_exact():
    g = gen.powerlaw_graph(4000, 100000, seed=41)
    g.val = np.random.default_rng(0).integers(1, 4, g.nnz).astype(np.float32)
    dg = upload(g)
    p = gs.plan(dg, 32)
    O = gs.spmm(p, dg, torch.ones((g.N, 32), device=DEV)).cpu().numpy()
    sums = np.bincount(g.row_ind, weights=g.val.astype(np.float64), minlength=g.M)
    assert np.array_equal(O.astype(np.float64), np.repeat(sums[:, None], 32, 1))


def test_sddmm_pair_symmetry_bitwise_and_self_loop_norm():
    g = gen.powerlaw_graph(3000, 50000, seed=42, val_mode="ones")
    dg = upload(g)
    K = 128
    X = torch.from_numpy(_x(42, g.N, K)).to(DEV)
    p = gs.plan(dg, K)
    out = gs.sddmm(p, dg, X, X).cpu().numpy()
    key = g.row_ind.astype(np.int64) * g.N + g.col_ind
    rkey = g.col_ind.astype(np.int64) * g.N + g.row_ind
    pos = np.searchsorted(key, rkey)
    assert np.array_equal(out, out[pos])  # (u,v) and (v,u) identical
    self_ = g.row_ind == g.col_ind
    Xn = X.cpu().numpy().astype(np.float64)
    nrm = (Xn ** 2).sum(1)[g.row_ind[self_]]
    assert np.allclose(out[self_], nrm, rtol=1e-5)


def test_fig4_fig5_worked_example():
    from test_oracle import fig4_matrix
    g, C, K, w, entries = fig4_matrix()
    dg = upload(g)
    p = gs.plan(dg, K, force_chunk=C)
    rf, rl, fl = (t.cpu().numpy() for t in p.arrays())
    assert (rf[w], rl[w]) == (3, 4)
    run_full(g, K, force_chunk=C)


# --------------------------------------------------------------- shards ----
@pytest.mark.parametrize("P", [2, 3, 8])
def test_virtual_row_and_edge_shards(P):
    """P shard plans run one after another on one GPU: row-sharded SpMM equals the
    unsharded result within tolerance, and edge-sharded SDDMM equals it bitwise (each
    output's dot product is computed in a fixed lane order whatever the chunking)."""
    g = gen.powerlaw_graph(6000, 300000, gamma=2.2, n_comm=6, seed=60 + P)
    K = 64
    A = _x(61, g.N, K)
    At = torch.from_numpy(A).to(DEV)
    dg = upload(g)
    ref, T = oracle.spmm(g.row_ind, g.col_ind, g.val, A, M=g.M)
    rb = gs.shard_rows(g.row_ptr, P)
    O = torch.empty((g.M, K), device=DEV)
    for q in range(P):
        r0, r1 = int(rb[q]), int(rb[q + 1])
        e0, e1 = int(g.row_ptr[r0]), int(g.row_ptr[r1])
        sh = dg.shard(r0, r1, e0, e1)
        p = gs.plan(sh, K)
        gs.spmm(p, sh, At, out=O[r0:r1])
    torch.cuda.synchronize()
    assert_within(O.cpu().numpy(), ref, T, what="row-sharded spmm")
    # edge shards for SDDMM
    full = gs.sddmm(gs.plan(dg, K), dg, At, At)
    eb = gs.shard_edges(g.nnz, P)
    out = torch.empty(g.nnz, device=DEV)
    for q in range(P):
        e0, e1 = int(eb[q]), int(eb[q + 1])
        sh = gs.DeviceGraph(g.M, g.N, dg.row_ind[e0:e1], dg.col_ind[e0:e1], dg.val[e0:e1])
        p = gs.plan(sh, K)
        gs.sddmm(p, sh, At, At, out=out[e0:e1])
    torch.cuda.synchronize()
    assert torch.equal(out, full)  # each output's dot is chunking-independent


def test_plan_spmm_sddmm_capture_in_cuda_graph():
    """No host sync anywhere on the path: plan + SpMM + SDDMM capture into a CUDA graph."""
    g = configs.make_c3(5)
    dg = upload(g)
    K = 128
    X = torch.from_numpy(_x(5, g.N, K)).to(DEV)
    O = torch.empty((g.M, K), device=DEV)
    E = torch.empty(g.nnz, device=DEV)
    nbytes = gs.lib().gnn_plan_workspace_bytes(g.M, g.nnz, K, None)
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    holder = []
    with torch.cuda.stream(s):
        gs.plan(dg, K)  # warm-up (occupancy cache) outside capture
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph, stream=s):
            p = gs.plan(dg, K)
            holder.append(p)
            gs.spmm(p, dg, X, out=O)
            gs.sddmm(p, dg, X, X, out=E)
    graph.replay()
    torch.cuda.synchronize()
    ref, T = oracle.spmm(g.row_ind, g.col_ind, g.val, X.cpu().numpy(), M=g.M)
    assert_within(O.cpu().numpy(), ref, T, what="graph-captured spmm")
    assert nbytes > 0


def test_misaligned_subview_falls_back_to_scalar_sparse_loads():
    g = gen.powerlaw_graph(4000, 200000, seed=77)
    dg = upload(g)
    r0 = 1
    e0 = int(g.row_ptr[r0])
    assert e0 % 4 != 0
    sh = dg.shard(r0, g.M, e0, g.nnz)
    K = 32
    A = _x(77, g.N, K)
    p = gs.plan(sh, K, force_chunk=128)
    assert p.info()["vw_sparse"] == 4
    O = gs.spmm(p, sh, torch.from_numpy(A).to(DEV))
    ref, T = oracle.spmm(g.row_ind, g.col_ind, g.val, A, i0=e0, i1=g.nnz, r0=r0, nrows=g.M - r0)
    assert_within(O.cpu().numpy(), ref, T, what="misaligned shard")


def test_unsupported_alignment_is_reported():
    g = gen.powerlaw_graph(500, 5000, seed=78)
    dg = upload(g)
    p = gs.plan(dg, 32)
    A = torch.zeros((g.N, 33), device=DEV)[:, 1:]  # 4-byte offset, pitch 33
    with pytest.raises(gs.GnnError) as e:
        gs.spmm(p, dg, A)
    assert e.value.status == gs.GNN_ERR_UNSUPPORTED


def test_graph_plan_mismatch_and_validate():
    g = gen.powerlaw_graph(500, 5000, seed=79)
    dg = upload(g)
    p = gs.plan(dg, 32)
    other = upload(gen.powerlaw_graph(500, 5000, seed=80))
    with pytest.raises(gs.GnnError):
        gs.spmm(p, other, torch.zeros((500, 32), device=DEV))
    gs.validate(dg)
    bad = gs.DeviceGraph(g.M, g.N, dg.row_ind.flip(0).contiguous(), dg.col_ind, dg.val)
    with pytest.raises(gs.GnnError) as e:
        gs.validate(bad)
    assert e.value.status == gs.GNN_ERR_INPUT_CHECK


def test_csr_to_coo_matches_oracle():
    g = gen.powerlaw_graph(7000, 90000, seed=81)
    rp = torch.from_numpy(g.row_ptr).to(DEV)
    ri = gs.csr_to_coo(rp).cpu().numpy()
    assert np.array_equal(ri, oracle.csr_to_coo(g.row_ptr))


def test_gcr_reordered_graph_equivariance():
    """SpMM(P S P^T, P X) = P SpMM(S, X) and SDDMM outputs move with their edges, on
    the GCR-reordered graph (gnn_reorder_gcr + gnn_permute_graph + gnn_permute_rows)."""
    g = gen.powerlaw_graph(20000, 400000, gamma=2.3, n_comm=20, mu=0.3, seed=5)
    perm, comm, q = gs.reorder_gcr(g.row_ptr, g.col_ind)
    rp, ri, ci, v = gs.permute_graph(g.row_ptr, g.col_ind, g.val, perm)
    gp = gen.Graph(g.M, g.N, rp, ri, ci, v)
    K = 64
    X = _x(70, g.N, K)
    Xd = torch.from_numpy(X).to(DEV)
    Xp = gs.permute_rows(Xd, torch.from_numpy(perm))
    torch.cuda.synchronize()
    assert torch.equal(Xp[torch.from_numpy(perm).long().to(DEV)], Xd)
    dgp = upload(gp)
    p = gs.plan(dgp, K)
    check_plan(p, gp, K)
    Op = gs.spmm(p, dgp, Xp).cpu().numpy()
    ref, T = oracle.spmm(g.row_ind, g.col_ind, g.val, X, M=g.M)
    assert_within(Op[perm], ref, T, what="reordered spmm")
    Ep = gs.sddmm(p, dgp, Xp, Xp).cpu().numpy()
    r2, T2 = oracle.sddmm(g.row_ind, g.col_ind, g.val, X, X)
    newkey = gp.row_ind.astype(np.int64) * g.N + gp.col_ind
    oldkey = perm[g.row_ind].astype(np.int64) * g.N + perm[g.col_ind]
    pos = np.searchsorted(newkey, oldkey)
    assert_within(Ep[pos], r2, T2, what="reordered sddmm")


# ------------------------------------------------- full BASELINE.json sizes ---
def _sampled_rows(g, n, seed):
    """A row sample that always includes the heaviest rows (hubs split across many
    chunks -> atomics), rows at chunk boundaries and random rows."""
    rng = np.random.default_rng(seed)
    deg = np.diff(g.row_ptr)
    heavy = np.argsort(deg)[-8:]
    rand = rng.choice(g.M, size=n, replace=False)
    return np.unique(np.r_[heavy, rand, 0, g.M - 1])


_FULL = {}


def full_graph(name, reorder):
    """Full-size BJ graph (C4 Reddit- / C5 products-shaped), GCR-reordered as bench.py
    runs it when reorder; cached for the module (generation + Louvain take ~10-20 s)."""
    key = (name, reorder)
    if key not in _FULL:
        g = configs.make_graph(name)
        perm = None
        if reorder:
            perm, _, _ = gs.reorder_gcr(g.row_ptr, g.col_ind)
            rp, ri, ci, v = gs.permute_graph(g.row_ptr, g.col_ind, g.val, perm)
            g = gen.Graph(g.M, g.N, rp, ri, ci, v)
        if len(_FULL) >= 2:
            _FULL.clear()
        _FULL[key] = (g, perm)
    return _FULL[key]


def _bench_features(name, g, K, perm):
    """bench.py's X for this K: the workload's features, rows relabelled by the GCR
    permutation (X' = P X)."""
    X = configs.make_features(name, g.N, K)
    if perm is not None:
        Xp = np.empty_like(X)
        Xp[perm] = X
        X = Xp
    return X


def _sampled_check(name, g, dg, p, X, Xd, K, tag, rows, edges, dtype=None):
    O = gs.spmm(p, dg, Xd)
    E = gs.sddmm(p, dg, Xd, Xd)
    torch.cuda.synchronize()
    ref, T = oracle.spmm_rows(g, X, rows)
    assert_within(O[torch.from_numpy(rows).to(DEV)].cpu().numpy(), ref, T,
                  what=f"{name} spmm K={K} {tag}")
    r2, T2 = oracle.sddmm_edges(g, X, X, edges)
    assert_within(E[torch.from_numpy(edges).to(DEV)].cpu().numpy(), r2, T2,
                  what=f"{name} sddmm K={K} {tag}")


@pytest.mark.slow
@pytest.mark.parametrize("name,Ks,reorder", [("C4", (32, 64, 128, 256), True),
                                             ("C4", (32, 256), False), ("C5", (256,), True)])
def test_full_size_sampled_parity(name, Ks, reorder):
    """Full-size Reddit / products-shaped graphs in bench.py's launch configuration
    (default plan; C4 GCR-reordered at every bench K, the headline config), checked on
    sampled output rows (SpMM) and edges (SDDMM) that the oracle computes one by one,
    plus the global plan arrays bit-exactly (device parameters derived independently)."""
    g, perm = full_graph(name, reorder)
    dg = upload(g)
    rows = _sampled_rows(g, 300, 1)
    edges = np.unique(np.r_[np.random.default_rng(2).choice(g.nnz, 20000, replace=False),
                            g.row_ptr[rows[:50]], g.nnz - 1])
    for K in Ks:
        X = _bench_features(name, g, K, perm)
        Xd = torch.from_numpy(X).to(DEV)
        p = gs.plan(dg, K)
        check_plan(p, g, K)
        _sampled_check(name, g, dg, p, X, Xd, K, "default plan", rows, edges)
        del Xd


@pytest.mark.slow
@pytest.mark.parametrize("name", ["C4", "C5"])
def test_full_size_paper_rule_plan(name):
    """The paper's DTP rule exactly (no_locality: InEq. 5 over the candidate set, no
    B200 cap / floor) at full C4 / C5 size: plan bit-exact with the oracle at every
    width bench.py runs, C* equal to the brute-force largest candidate with >= alpha full
    waves, and outputs within the bar on samples under that plan."""
    g, perm = full_graph(name, True)
    dg = upload(g)
    rows = _sampled_rows(g, 150, 5)
    edges = np.unique(np.random.default_rng(6).choice(g.nnz, 5000, replace=False))
    Ks = (32, 64, 128, 256) if name == "C4" else (256,)
    for K in Ks:
        p = gs.plan(dg, K, no_locality=True)
        info = check_plan(p, g, K, no_locality=True)
        FW = info["num_sms"] * info["active_blocks_per_sm"]
        S, G, W = info["slices"], info["groups"], info["warps_per_block"]
        cdiv = lambda a, b: -(-a // b)
        blocks = lambda C: cdiv(cdiv(cdiv(g.nnz, C) * S, G), W)  # InEq. 5 RHS
        ok = [C for C in (8, 32, 64, 128, 256, 512) if blocks(C) >= 2 * FW]
        assert info["chunk"] == info["chunk_dtp"] == (max(ok) if ok else 8)
        if K in (32, 256):
            X = _bench_features(name, g, K, perm)
            Xd = torch.from_numpy(X).to(DEV)
            _sampled_check(name, g, dg, p, X, Xd, K, "paper rule", rows, edges)
            del Xd


@pytest.mark.slow
def test_full_size_bf16_bench_config():
    """bench.py's bf16 leg at full size (C4, GCR, K = 32 and 256): exact-input parity
    (the oracle gets the bf16 values) on samples."""
    g, perm = full_graph("C4", True)
    dg = upload(g)
    rows = _sampled_rows(g, 150, 7)
    edges = np.unique(np.random.default_rng(8).choice(g.nnz, 5000, replace=False))
    for K in (32, 256):
        Xb = torch.from_numpy(_bench_features("C4", g, K, perm)).to(torch.bfloat16)
        X = Xb.float().numpy()
        p = gs.plan(dg, K, feature_dtype="bf16")
        check_plan(p, g, K, feature_dtype="bf16")
        _sampled_check("C4", g, dg, p, X, Xb.to(DEV), K, "bf16", rows, edges)


# ------------------------------------------------------------ bf16 (f2) ----
def _bf16_pair(seed, rows, K):
    """bf16 features (round-to-nearest-even of the fp32 generator) and their exact fp32
    values (bf16 -> fp32 widening is exact)."""
    X = torch.from_numpy(_x(seed, rows, K))
    Xb = X.to(torch.bfloat16)
    return Xb.to(DEV), Xb.float().numpy(), X.numpy()


@pytest.mark.parametrize("K", [2, 6, 24, 32, 64, 128, 256, 512])
def test_bf16_features_parity(K):
    """bf16 gathered features, fp32 accumulation: exact-input parity within 1e-5 * T
    (the oracle is fed the bf16 values), and within 1e-2 * T of the fp32-feature result
    (BASELINE.json bf16 bar)."""
    g = gen.powerlaw_graph(4000, 120000, gamma=2.2, n_comm=6, seed=500 + K)
    dg = upload(g)
    p = gs.plan(dg, K, feature_dtype="bf16")
    check_plan(p, g, K, feature_dtype="bf16")
    Xb, Xexact, X32 = _bf16_pair(600 + K, g.N, K)
    A1b, A1exact, A132 = _bf16_pair(700 + K, g.M, K)
    O = gs.spmm(p, dg, Xb).cpu().numpy()
    E = gs.sddmm(p, dg, A1b, Xb).cpu().numpy()
    r, T = oracle.spmm(g.row_ind, g.col_ind, g.val, Xexact, M=g.M)
    assert_within(O, r, T, what=f"bf16 spmm K={K} (exact inputs)")
    r32, T32 = oracle.spmm(g.row_ind, g.col_ind, g.val, X32, M=g.M)
    assert_within(O, r32, T32, tol=1e-2, what=f"bf16 spmm K={K} vs fp32")
    r2, T2 = oracle.sddmm(g.row_ind, g.col_ind, g.val, A1exact, Xexact)
    assert_within(E, r2, T2, what=f"bf16 sddmm K={K} (exact inputs)")
    r232, T232 = oracle.sddmm(g.row_ind, g.col_ind, g.val, A132, X32)
    assert_within(E, r232, T232, tol=1e-2, what=f"bf16 sddmm K={K} vs fp32")


def test_bf16_plan_dtype_mismatch_rejected():
    g = gen.powerlaw_graph(500, 5000, seed=510)
    dg = upload(g)
    p = gs.plan(dg, 32)  # fp32 plan
    with pytest.raises(gs.GnnError):
        gs.spmm(p, dg, torch.zeros((g.N, 32), dtype=torch.bfloat16, device=DEV))


@pytest.mark.parametrize("P", [2, 4, 8])
def test_column_block_accumulation_equals_spmm(P):
    """f1 building block: a row shard split by column owner block (gnn_split_col_blocks),
    SpMM of the local block (beta = 0) then the others accumulated (beta = 1) in
    block_order, equals the shard's SpMM."""
    from paper_conf_ipps_fanwc23_b200 import dist as gdist
    g = gen.powerlaw_graph(6000, 300000, gamma=2.2, n_comm=6, seed=90 + P)
    K = 64
    X = _x(91, g.N, K)
    for rank in range(P):
        s = gdist.shard_spec(g.row_ptr, g.N, rank, P)
        ro, co, vo, b = gs.split_col_blocks(g.row_ind[s.e0:s.e1], g.col_ind[s.e0:s.e1],
                                            g.val[s.e0:s.e1], P, s.xblk)
        Xf = np.zeros((s.xblk * P, K), np.float32)
        Xf[:g.N] = X
        Xd = torch.from_numpy(Xf).to(DEV)
        O = torch.full((s.r1 - s.r0, K), float("nan"), device=DEV)
        first = True
        for q in gdist.block_order(P, rank):
            a, z = int(b[q]), int(b[q + 1])
            bg = gs.DeviceGraph.from_arrays(s.r1 - s.r0, s.xblk * P, ro[a:z], co[a:z], vo[a:z],
                                            row_base=s.r0)
            gs.spmm(gs.plan(bg, K), bg, Xd, out=O, accumulate=not first)
            first = False
        ref, T = oracle.spmm(g.row_ind, g.col_ind, g.val, X, i0=s.e0, i1=s.e1, r0=s.r0,
                             nrows=s.r1 - s.r0)
        torch.cuda.synchronize()
        assert_within(O.cpu().numpy(), ref, T, what=f"column blocks P={P} rank={rank}")


def test_run_host_end_to_end_matches_oracle():
    """gnn_run_host (HOST buffers in, HOST results out) for several K with one workspace
    and one graph upload."""
    g = configs.make_graph("C2")
    runner = gs.HostRunner(g.M, g.N, g.row_ind, g.col_ind, g.val, 128, device=DEV).pin()
    for j, K in enumerate((32, 64, 128)):
        X = torch.from_numpy(_x(800 + K, g.N, K)).pin_memory()
        O = torch.empty((g.M, K)).pin_memory()
        E = torch.empty(g.nnz).pin_memory()
        runner.run(X, K, O, E, upload_graph=(j == 0))
        torch.cuda.synchronize()
        ref, T = oracle.spmm(g.row_ind, g.col_ind, g.val, X.numpy(), M=g.M)
        assert_within(O.numpy(), ref, T, what=f"run_host spmm K={K}")
        r2, T2 = oracle.sddmm(g.row_ind, g.col_ind, g.val, X.numpy(), X.numpy())
        assert_within(E.numpy(), r2, T2, what=f"run_host sddmm K={K}")


def _run_host_check(g, Ks, pieces, seed=900, opts=None, csr=False):
    """gnn_run_host with GNN_HOST_PIECES=pieces against the oracle everywhere (csr: the
    graph goes up as CSR offsets, RowInd decoded on the device)."""
    import os
    old = os.environ.get("GNN_HOST_PIECES")
    os.environ["GNN_HOST_PIECES"] = str(pieces)
    try:
        runner = gs.HostRunner(g.M, g.N, g.row_ind, g.col_ind, g.val, max(Ks), device=DEV,
                               row_ptr=g.row_ptr if csr else None, **(opts or {})).pin()
        for j, K in enumerate(Ks):
            X = torch.from_numpy(_x(seed + K, g.N, K)).pin_memory()
            O = torch.full((g.M, K), float("nan")).pin_memory()
            E = torch.full((g.nnz,), float("nan")).pin_memory()
            runner.run(X, K, O, E, upload_graph=(j == 0))
            torch.cuda.synchronize()
            ref, T = oracle.spmm(g.row_ind, g.col_ind, g.val, X.numpy(), M=g.M)
            assert_within(O.numpy(), ref, T, what=f"run_host pieces={pieces} spmm K={K}")
            r2, T2 = oracle.sddmm(g.row_ind, g.col_ind, g.val, X.numpy(), X.numpy())
            assert_within(E.numpy(), r2, T2, what=f"run_host pieces={pieces} sddmm K={K}")
    finally:
        if old is None:
            del os.environ["GNN_HOST_PIECES"]
        else:
            os.environ["GNN_HOST_PIECES"] = old


@pytest.mark.parametrize("csr", [False, True])
@pytest.mark.parametrize("pieces", [2, 3, 7, 32])
def test_run_host_pipelined_pieces(pieces, csr):
    """The copy/compute pipeline of gnn_run_host (pieces of the plan's chunks on two
    compute streams, O rows downloaded as they become final): every output element
    matches the oracle for any piece count, including pieces whose boundaries fall
    inside a row, before runs of empty rows and inside a hub row; with the graph uploaded
    as RowInd or as CSR offsets decoded on the device."""
    g = configs.make_graph("C2")
    _run_host_check(g, (32, 64, 256), pieces, csr=csr)
    rng = np.random.default_rng(17)
    M = 3000
    rows = rng.integers(0, M, 60000)
    rows = rows[(rows % 11) > 2]  # runs of empty rows
    rows = np.concatenate([rows, np.full(20000, 1500), [0, M - 1]])  # hub + first/last row
    cols = rng.integers(0, M, rows.size)
    g2 = gen.from_coo(M, M, rows, cols, gen.uniform_values(5, rows.size))
    _run_host_check(g2, (8, 32, 128), pieces, csr=csr)


@pytest.mark.parametrize("chunk", [1000, 4096])
def test_run_host_pieces_smaller_than_chunks(chunk):
    """Pieces are ranges of nonzeros common to every width and a width takes the chunks
    that end inside a piece: with chunks longer than a piece, some pieces run no chunk of
    that width, and a chunk's plan entry (tail flag) reads the first row of the next piece."""
    g = configs.make_graph("C2")
    _run_host_check(g, (32, 64), 32, opts={"force_chunk": chunk})


def test_run_host_pipelined_deterministic_and_no_values():
    """Deterministic plans run unpipelined; a NULL value array means all ones."""
    g = configs.make_graph("C2")
    _run_host_check(g, (64,), 8, opts={"deterministic": 1})
    g1 = gen.Graph(g.M, g.N, g.row_ptr, g.row_ind, g.col_ind, None)
    _run_host_check(g1, (32, 128), 5)


@pytest.mark.slow
def test_run_host_full_size_sampled_parity():
    """bench.py's e2e call at full C4 size (default piece count, graph uploaded by the
    first K, reused by the second): sampled rows / edges against the oracle."""
    g = configs.make_graph("C4")
    runner = gs.HostRunner(g.M, g.N, g.row_ind, g.col_ind, g.val, 256, device=DEV).pin()
    rows = _sampled_rows(g, 200, 3)
    edges = np.unique(np.r_[np.random.default_rng(4).choice(g.nnz, 5000, replace=False),
                            g.row_ptr[rows[:50]], g.nnz - 1])
    for j, K in enumerate((32, 256)):
        X = configs.make_features("C4", g.N, K)
        O = torch.empty((g.M, K)).pin_memory()
        E = torch.empty(g.nnz).pin_memory()
        runner.run(torch.from_numpy(X).pin_memory(), K, O, E, upload_graph=(j == 0))
        torch.cuda.synchronize()
        ref, T = oracle.spmm_rows(g, X, rows)
        assert_within(O.numpy()[rows], ref, T, what=f"run_host C4 spmm K={K}")
        r2 = np.empty(edges.size)
        T2 = np.empty(edges.size)
        for i, e in enumerate(edges):
            a, b = oracle.sddmm(g.row_ind, g.col_ind, g.val, X, X, i0=int(e), i1=int(e) + 1)
            r2[i], T2[i] = a[0], b[0]
        assert_within(E.numpy()[edges], r2, T2, what=f"run_host C4 sddmm K={K}")


@pytest.mark.slow
def test_run_host_multi_full_size_bench_config():
    """bench.py's e2e headline exactly: one gnn_run_host_multi call over K = 32..256 on
    the GCR-reordered full C4 graph with the default piece count, NaN-prefilled pinned
    outputs; sampled rows / edges of every width against the oracle (and no element of
    any output left unwritten)."""
    g, perm = full_graph("C4", True)
    Ks = (32, 64, 128, 256)
    runner = gs.HostRunner(g.M, g.N, g.row_ind, g.col_ind, g.val, max(Ks), device=DEV,
                           Ks=Ks, row_ptr=g.row_ptr).pin()  # CSR upload, as bench.py
    Xs = [torch.from_numpy(_bench_features("C4", g, K, perm)).pin_memory() for K in Ks]
    Os = [torch.full((g.M, K), float("nan")).pin_memory() for K in Ks]
    Es = [torch.full((g.nnz,), float("nan")).pin_memory() for _ in Ks]
    runner.run_multi(Xs, Ks, Os, Es, upload_graph=True)
    torch.cuda.synchronize()
    rows = _sampled_rows(g, 200, 9)
    edges = np.unique(np.r_[np.random.default_rng(10).choice(g.nnz, 5000, replace=False),
                            g.row_ptr[rows[:50]], g.nnz - 1])
    for j, K in enumerate(Ks):
        assert not torch.isnan(Os[j]).any() and not torch.isnan(Es[j]).any(), K
        X = Xs[j].numpy()
        ref, T = oracle.spmm_rows(g, X, rows)
        assert_within(Os[j].numpy()[rows], ref, T, what=f"run_host_multi C4 spmm K={K}")
        r2, T2 = oracle.sddmm_edges(g, X, X, edges)
        assert_within(Es[j].numpy()[edges], r2, T2, what=f"run_host_multi C4 sddmm K={K}")


def _run_multi_check(g, Ks, pieces=None, skip_o=(), seed=950, csr=False):
    """gnn_run_host_multi over several widths in one call, every output vs the oracle."""
    import os
    old = os.environ.get("GNN_HOST_PIECES")
    if pieces is not None:
        os.environ["GNN_HOST_PIECES"] = str(pieces)
    try:
        runner = gs.HostRunner(g.M, g.N, g.row_ind, g.col_ind, g.val, max(Ks), device=DEV,
                               Ks=Ks, row_ptr=g.row_ptr if csr else None).pin()
        Xs = [torch.from_numpy(_x(seed + K, g.N, K)).pin_memory() for K in Ks]
        Os = [None if j in skip_o else torch.full((g.M, K), float("nan")).pin_memory()
              for j, K in enumerate(Ks)]
        Es = [torch.full((g.nnz,), float("nan")).pin_memory() for _ in Ks]
        for rep in range(2):  # the second call reuses the uploaded graph
            runner.run_multi(Xs, Ks, Os, Es, upload_graph=(rep == 0))
            torch.cuda.synchronize()
            for j, K in enumerate(Ks):
                X = Xs[j].numpy()
                if Os[j] is not None:
                    ref, T = oracle.spmm(g.row_ind, g.col_ind, g.val, X, M=g.M)
                    assert_within(Os[j].numpy(), ref, T, what=f"multi spmm K={K} rep={rep}")
                r2, T2 = oracle.sddmm(g.row_ind, g.col_ind, g.val, X, X)
                assert_within(Es[j].numpy(), r2, T2, what=f"multi sddmm K={K} rep={rep}")
                Es[j].fill_(float("nan"))
                if Os[j] is not None:
                    Os[j].fill_(float("nan"))
    finally:
        if old is None:
            os.environ.pop("GNN_HOST_PIECES", None)
        else:
            os.environ["GNN_HOST_PIECES"] = old


@pytest.mark.parametrize("csr", [False, True])
@pytest.mark.parametrize("pieces", [None, 3, 32])
def test_run_host_multi_widths(pieces, csr):
    """Several feature widths in one pipelined gnn_run_host_multi call (per-width plans,
    pieces alternating over two compute streams across widths, one width's SpMM skipped;
    graph uploaded as RowInd or as CSR offsets)."""
    g = configs.make_graph("C2")
    _run_multi_check(g, (32, 8, 256, 64), pieces, skip_o=(1,), csr=csr)
    rng = np.random.default_rng(23)
    M = 2500
    rows = rng.integers(0, M, 50000)
    rows = rows[(rows % 13) > 3]
    rows = np.concatenate([rows, np.full(15000, 700), [M - 1]])
    g2 = gen.from_coo(M, M, rows, rng.integers(0, M, rows.size), gen.uniform_values(6, rows.size))
    _run_multi_check(g2, (16, 128), pieces, csr=csr)


def test_run_host_multi_rejects_bad_arguments():
    g = configs.make_graph("C1")
    runner = gs.HostRunner(g.M, g.N, g.row_ind, g.col_ind, g.val, 32, device=DEV, Ks=(32,))
    X = torch.zeros((g.N, 32))
    with pytest.raises(gs.GnnError):
        runner.run_multi([X], [0])
    with pytest.raises(gs.GnnError):
        runner.run_multi([X] * 17, [32] * 17)


@pytest.mark.parametrize("no_locality", [False, True])
def test_locality_cap_plan_and_parity(no_locality):
    """A low-degree graph with wide rows, where the L2 locality cap (DESIGN.md §3 step
    5b) lowers C* below the DTP choice: plan info and arrays bit-exact with the oracle
    (which is given the device's L2 size), outputs within the fp32 bar; with
    no_locality the plain DTP choice is kept."""
    rng = np.random.default_rng(31)
    M = 200_000
    # 3.2 M nonzeros (degree 16): DTP picks 128-512 and the cap 64-128 (the step-5c floor
    # of 64 leaves the cap visible; 0.8 M nonzeros had DTP itself at 64)
    rows = np.sort(rng.integers(0, M, 3_200_000))
    g = gen.from_coo(M, M, rows, rng.integers(0, M, rows.size), gen.uniform_values(8, rows.size))
    info, _ = run_full(g, 256, no_locality=no_locality)
    if no_locality:
        assert info["chunk"] == info["chunk_dtp"]
    else:
        assert info["chunk"] < info["chunk_dtp"]


def test_run_host_multi_row_shards():
    """gnn_run_host_multi on nnz-balanced row shards (bench.py's e2e at N ranks): each
    shard's O rows and S_O entries (A1 = the shard's rows of X) against the oracle."""
    import os
    g = configs.make_graph("C2")
    Ks = (32, 128)
    Xs = [torch.from_numpy(_x(990 + K, g.N, K)).pin_memory() for K in Ks]
    os.environ["GNN_HOST_PIECES"] = "4"
    try:
        for P in (2, 3):
            b = gs.shard_rows(g.row_ptr, P)
            for p in range(P):
                r0, r1 = int(b[p]), int(b[p + 1])
                e0, e1 = int(g.row_ptr[r0]), int(g.row_ptr[r1])
                runner = gs.HostRunner(r1 - r0, g.N, g.row_ind[e0:e1], g.col_ind[e0:e1],
                                       g.val[e0:e1], max(Ks), device=DEV, Ks=Ks,
                                       row_base=r0,
                                       row_ptr=g.row_ptr[r0:r1 + 1] if p % 2 else None).pin()
                Os = [torch.full((r1 - r0, K), float("nan")).pin_memory() for K in Ks]
                Es = [torch.full((e1 - e0,), float("nan")).pin_memory() for _ in Ks]
                runner.run_multi(Xs, Ks, Os, Es)
                torch.cuda.synchronize()
                for j, K in enumerate(Ks):
                    X = Xs[j].numpy()
                    ref, T = oracle.spmm(g.row_ind, g.col_ind, g.val, X, i0=e0, i1=e1, r0=r0,
                                         nrows=r1 - r0)
                    assert_within(Os[j].numpy(), ref, T, what=f"shard {p}/{P} spmm K={K}")
                    r2, T2 = oracle.sddmm(g.row_ind, g.col_ind, g.val, X, X, i0=e0, i1=e1)
                    assert_within(Es[j].numpy(), r2, T2, what=f"shard {p}/{P} sddmm K={K}")
    finally:
        os.environ.pop("GNN_HOST_PIECES", None)


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
def test_feature_matrix_beyond_4GB(dtype):
    """Byte offsets of gathered rows beyond 2^32 (X of 4.6 GB: row c starts at c * 1 KB
    (fp32) / 512 B (bf16) with K = 256): the 64-bit address arithmetic of both kernels.
    300 destination rows gather from the last rows of X and from random ones; the oracle
    sees only the referenced rows (counter-based features: the same values by row id)."""
    K = 256
    N = 4_500_000 if dtype == "f32" else 9_000_000
    M, deg, seed = 300, 160, 4242
    rng = np.random.default_rng(77)
    rows = np.repeat(np.arange(M), deg)
    cols = np.where(rng.random(rows.size) < 0.5, rng.integers(N - 200_000, N, rows.size),
                    rng.integers(0, N, rows.size))
    g = gen.from_coo(M, N, rows, cols, gen.uniform_values(78, rows.size))
    dg = upload(g)
    X = torch.empty((N, K), dtype=torch.float32 if dtype == "f32" else torch.bfloat16, device=DEV)
    step = 1_000_000
    for r0 in range(0, N, step):
        n = min(step, N - r0)
        X[r0:r0 + n] = torch.from_numpy(gen.features(seed, n, K, row0=r0)).to(DEV)
    assert X.numel() * X.element_size() > (1 << 32)
    p = gs.plan(dg, K, feature_dtype=dtype)
    O = gs.spmm(p, dg, X).cpu().numpy()
    E = gs.sddmm(p, dg, X, X).cpu().numpy()
    # the oracle on the referenced rows only (column ids remapped); bf16: the rounded values
    uniq, inv = np.unique(np.concatenate([g.col_ind, np.arange(M)]), return_inverse=True)
    Xs = np.concatenate([gen.features(seed, 1, K, row0=int(c)) for c in uniq])
    if dtype == "bf16":
        Xs = torch.from_numpy(Xs).to(torch.bfloat16).float().numpy()
    col_s = inv[:g.nnz].astype(np.int32)
    A1s = Xs[inv[g.nnz:]]
    r, T = oracle.spmm(g.row_ind, col_s, g.val, Xs, M=M)
    assert_within(O, r, T, what=f"spmm {dtype} X > 4 GB")
    r2, T2 = oracle.sddmm(g.row_ind, col_s, g.val, A1s, Xs)
    assert_within(E, r2, T2, what=f"sddmm {dtype} X > 4 GB")


def test_plan_spmm_sddmm_one_call():
    """gnn_plan_spmm_sddmm (plan + SpMM + SDDMM with A1 = A2T = X in one native call, the
    SDDMM on a forked side stream; the plan workspace reused across graphs): every output
    against the oracle on sampled subgraphs of different sizes, a row shard (row_base > 0,
    A1 = the shard's rows of X) and the single-output forms."""
    run = gs.StepRunner()
    for t in (0, 1, 2, 0):
        g = configs.make_c3(t)
        dg = upload(g)
        X = _x(960 + t, g.N, 128)
        Xd = torch.from_numpy(X).to(DEV)
        O = torch.full((g.M, 128), float("nan"), device=DEV)
        E = torch.full((g.nnz,), float("nan"), device=DEV)
        run(dg, Xd, O, E)
        torch.cuda.synchronize()
        r, T = oracle.spmm(g.row_ind, g.col_ind, g.val, X, M=g.M)
        assert_within(O.cpu().numpy(), r, T, what=f"one-call spmm t={t}")
        r2, T2 = oracle.sddmm(g.row_ind, g.col_ind, g.val, X, X)
        assert_within(E.cpu().numpy(), r2, T2, what=f"one-call sddmm t={t}")
    # row shard [r0, r1) of a square graph
    g = configs.make_graph("C2")
    r0, r1 = 5000, 12000
    e0, e1 = int(g.row_ptr[r0]), int(g.row_ptr[r1])
    full = upload(g)
    sh = full.shard(r0, r1, e0, e1)
    X = _x(970, g.N, 64)
    Xd = torch.from_numpy(X).to(DEV)
    O = torch.full((r1 - r0, 64), float("nan"), device=DEV)
    E = torch.full((e1 - e0,), float("nan"), device=DEV)
    run(sh, Xd, O, E)
    torch.cuda.synchronize()
    r, T = oracle.spmm(g.row_ind, g.col_ind, g.val, X, i0=e0, i1=e1, r0=r0, nrows=r1 - r0)
    assert_within(O.cpu().numpy(), r, T, what="one-call spmm shard")
    r2, T2 = oracle.sddmm(g.row_ind, g.col_ind, g.val, X, X, i0=e0, i1=e1)
    assert_within(E.cpu().numpy(), r2, T2, what="one-call sddmm shard")
    # one output only
    E2 = torch.full((e1 - e0,), float("nan"), device=DEV)
    run(sh, Xd, None, E2)
    O2 = torch.full((r1 - r0, 64), float("nan"), device=DEV)
    run(sh, Xd, O2, None)
    torch.cuda.synchronize()
    assert torch.equal(E2, E)  # SDDMM writes each output once: bit-reproducible
    assert_within(O2.cpu().numpy(), r, T, what="one-call spmm only")  # (atomics: not bitwise)


def test_binding_rejects_undersized_or_mistyped_operands():
    """The Python layer checks every dense operand's dtype, shape and device before a
    pointer reaches a kernel (an undersized tensor would be read / written out of
    bounds)."""
    g = configs.make_graph("C1")
    dg = upload(g)
    K = 32
    p = gs.plan(dg, K)
    X = torch.zeros((g.N, K), device=DEV)
    bad = [lambda: gs.spmm(p, dg, X[: g.N - 1]),
           lambda: gs.spmm(p, dg, torch.zeros((g.N, K - 8), device=DEV)),
           lambda: gs.spmm(p, dg, X, out=torch.empty((g.M - 1, K), device=DEV)),
           lambda: gs.sddmm(p, dg, X[: g.M - 1], X),
           lambda: gs.sddmm(p, dg, X, X, out=torch.empty(g.nnz - 1, device=DEV)),
           lambda: gs.sddmm(p, dg, X, X, out=torch.empty(g.nnz, dtype=torch.float64,
                                                          device=DEV)),
           lambda: gs.StepRunner(DEV)(dg, X.to(torch.bfloat16), None,
                                      torch.empty(g.nnz, device=DEV)),
           lambda: gs.StepRunner(DEV)(dg, X, torch.empty((g.M, K - 8), device=DEV), None),
           lambda: gs.StepRunner(DEV)(dg, X, None, torch.empty(g.nnz - 1, device=DEV))]
    for f in bad:
        with pytest.raises(ValueError):
            f()


def test_validate_env_switch(monkeypatch):
    """GNN_VALIDATE=1 makes gnn_plan_create check the graph first (a decreasing row_ind
    is reported as GNN_ERR_INPUT_CHECK); unset, the same call plans without a check."""
    g = configs.make_graph("C1")
    ri = g.row_ind.copy()
    ri[10], ri[11] = ri[11] + 1, ri[10]  # not non-decreasing
    dg = gs.DeviceGraph.from_arrays(g.M, g.N, ri, g.col_ind, g.val, None, device=DEV)
    monkeypatch.setenv("GNN_VALIDATE", "1")
    with pytest.raises(gs.GnnError) as e:
        gs.plan(dg, 32)
    assert e.value.status == 5
    monkeypatch.delenv("GNN_VALIDATE")
    gs.plan(dg, 32)


@pytest.mark.parametrize("mode", ["fused", "two_kernels", "plan_kernel"])
def test_one_call_step_inline_plan_matches_oracle(monkeypatch, mode):
    """gnn_plan_spmm_sddmm against the oracle on graphs with hubs split over many chunks
    and empty rows, in its three forms: one fused SpMM+SDDMM launch (default), the two
    kernels on two streams (GNN_STEP_FUSED=0), both with the boundary table recomputed in
    the kernels and a PDL SpMM, and the plan-kernel path (GNN_STEP_PLAN_KERNEL=1)."""
    monkeypatch.setenv("GNN_STEP_FUSED", "0" if mode == "two_kernels" else "1")
    monkeypatch.setenv("GNN_STEP_PLAN_KERNEL", "1" if mode == "plan_kernel" else "0")
    rng = np.random.default_rng(77)
    for t in range(6):
        M = int(rng.integers(100, 3000))
        nnz = int(rng.integers(1000, 60000))
        rows = np.sort(rng.integers(0, M, nnz))
        rows[: nnz // 4] = rows[0]  # a hub
        g = gen.from_coo(M, M, rows, rng.integers(0, M, nnz), gen.uniform_values(80 + t, nnz))
        K = int(rng.choice([32, 64, 128, 256])) if t else 24  # (24: no fused instance)
        dg = upload(g)
        X = torch.from_numpy(_x(90 + t, g.N, K)).to(DEV)
        O = torch.full((g.M, K), float("nan"), device=DEV)
        E = torch.full((g.nnz,), float("nan"), device=DEV)
        gs.StepRunner(DEV)(dg, X, O, E)
        torch.cuda.synchronize()
        Xh = X.cpu().numpy()
        ref, T = oracle.spmm(g.row_ind, g.col_ind, g.val, Xh, M=g.M)
        assert_within(O.cpu().numpy(), ref, T, what=f"one-call spmm t={t}")
        r2, T2 = oracle.sddmm(g.row_ind, g.col_ind, g.val, Xh, Xh)
        assert_within(E.cpu().numpy(), r2, T2, what=f"one-call sddmm t={t}")


def test_subnormal_partials_atomic_ftz_vs_deterministic():
    """Documented limit (reading 28, device.cuh): the vector atomics that combine a
    row split across chunks (REDG.E.ADD.F32x4) flush subnormal operands to zero.  With
    subnormal features a split row may lose its partial sums on the default plan, while
    rows owned by one chunk are exact; a deterministic plan (split rows summed in chunk
    order by plain fp32 adds, no atomics) keeps them: exact here (sums of subnormals are
    exact until they leave the subnormal range)."""
    M = N = 64
    rows = np.r_[np.zeros(2000, np.int64), np.repeat(np.arange(1, M), 3)]
    rng = np.random.default_rng(5)
    g = gen.from_coo(M, N, rows, rng.integers(0, N, rows.size), np.ones(rows.size, np.float32))
    K = 32
    X = (rng.integers(1, 4, (N, K)).astype(np.float64) * 2.0 ** -140).astype(np.float32)
    assert (X != 0).all() and (np.abs(X) < np.finfo(np.float32).tiny).all()  # subnormal
    ref, T = oracle.spmm(g.row_ind, g.col_ind, g.val, X, M=g.M)
    dg = upload(g)
    Xd = torch.from_numpy(X).to(DEV)
    det = gs.spmm(gs.plan(dg, K, deterministic=True), dg, Xd).cpu().numpy()
    assert np.array_equal(det.astype(np.float64), ref)
    p = gs.plan(dg, K)
    C = p.info()["chunk"]
    first, last = g.row_ptr[:-1] // C, (g.row_ptr[1:] - 1) // C
    split = first != last                                     # rows spanning chunks
    assert split[0]
    O = gs.spmm(p, dg, Xd).cpu().numpy().astype(np.float64)
    assert np.array_equal(O[~split], ref[~split])             # rows owned by one chunk
    assert (O[split] >= 0).all() and (O[split] <= ref[split]).all()  # flushed partials
