"""GPU parity for the NEXT rows f3/f4: aggregators (Eq. 1 with
(+) in {sum, mean, max, min}), beta = 1 accumulation, the device transpose, the autograd
backward pair (dX = S^T dO, dv = SDDMM(dO, X)) and a GCN training smoke test."""
import numpy as np
import pytest
import torch

import gen
import oracle
import paper_conf_ipps_fanwc23_b200 as gs
from paper_conf_ipps_fanwc23_b200 import nn as gnn

from helpers import oracle_plan_checked, assert_within, upload

pytestmark = pytest.mark.gpu
DEV = "cuda"


def graphs():
    rng = np.random.default_rng(7)
    M, N = 900, 700
    rows = rng.integers(0, M, 30000)
    rows = rows[(rows % 9) != 4]                       # empty rows
    rows = np.concatenate([rows, np.full(6000, 17)])   # a hub split across many chunks
    cols = rng.integers(0, N, rows.size)
    vals = rng.uniform(-1, 1, rows.size).astype(np.float32)
    yield gen.from_coo(M, N, rows, cols, vals)
    yield gen.powerlaw_graph(5000, 150000, gamma=2.2, n_comm=5, seed=8)


@pytest.mark.parametrize("agg", ["sum", "mean", "max", "min"])
@pytest.mark.parametrize("K", [8, 32, 64, 256])
@pytest.mark.parametrize("C", [0, 8, 64])
def test_spmm_aggregators(agg, K, C):
    for g in graphs():
        dg = upload(g)
        p = gs.plan(dg, K, force_chunk=C)
        X = gen.features(31 + K, g.N, K)
        O = gs.spmm(p, dg, torch.from_numpy(X).to(DEV), agg=agg).cpu().numpy()
        ref, T = oracle.spmm_agg(g.row_ind, g.col_ind, g.val, X, agg, M=g.M)
        tol = 1e-5 if agg in ("sum", "mean") else 1e-6   # max/min: one rounded product
        assert_within(O, ref, T, tol=tol, what=f"{agg} K={K} C={C}")


def test_spmm_accumulate_beta_one():
    g = gen.powerlaw_graph(3000, 60000, seed=9)
    dg = upload(g)
    K = 64
    p = gs.plan(dg, K)
    X = gen.features(40, g.N, K)
    O0 = gen.features(41, g.M, K)
    O = torch.from_numpy(O0.copy()).to(DEV)
    gs.spmm(p, dg, torch.from_numpy(X).to(DEV), out=O, accumulate=True)
    ref, T = oracle.spmm(g.row_ind, g.col_ind, g.val, X, M=g.M)
    assert_within(O.cpu().numpy(), ref + O0.astype(np.float64), T + np.abs(O0), what="beta=1")


def test_transpose_matches_definition():
    for g in graphs():
        dg = upload(g)
        gt, perm = gs.transpose(dg)
        order = np.lexsort((np.arange(g.nnz), g.row_ind, g.col_ind))  # by col, row, stable
        assert np.array_equal(perm.cpu().numpy(), order)
        assert np.array_equal(gt.row_ind.cpu().numpy(), g.col_ind[order])
        assert np.array_equal(gt.col_ind.cpu().numpy(), g.row_ind[order])
        assert np.array_equal(gt.val.cpu().numpy(), g.val[order])
        cnt = np.bincount(g.col_ind, minlength=g.N)
        assert np.array_equal(gt.row_ptr.cpu().numpy(), np.r_[0, np.cumsum(cnt)])


@pytest.mark.parametrize("agg", ["sum", "mean"])
def test_autograd_backward_pair(agg):
    """loss = <G, SpMM(S, X)>: dX = S^T G (mean: S^T (G / cnt)) and dv_i = <G_r, X_c>."""
    for g in graphs():
        dg = upload(g)
        op = gnn.SparseOp(dg)
        K = 32
        X = torch.from_numpy(gen.features(50, g.N, K)).to(DEV).requires_grad_(True)
        val = torch.from_numpy(g.val.copy()).to(DEV).requires_grad_(True)
        G = gen.features(51, g.M, K)
        O = gnn.spmm_autograd(op, X, val, agg=agg)
        (O * torch.from_numpy(G).to(DEV)).sum().backward()
        cnt = np.diff(g.row_ptr).astype(np.float64)
        Gs = (G / np.maximum(cnt, 1)[:, None]).astype(np.float32) if agg == "mean" else G
        order = np.lexsort((np.arange(g.nnz), g.row_ind, g.col_ind))
        dX_ref, TdX = oracle.spmm(g.col_ind[order], g.row_ind[order], g.val[order], Gs, M=g.N)
        assert_within(X.grad.cpu().numpy(), dX_ref, TdX, what=f"dX ({agg})")
        dv_ref, Tdv = oracle.sddmm(g.row_ind, g.col_ind, None, Gs, X.detach().cpu().numpy())
        assert_within(val.grad.cpu().numpy(), dv_ref, Tdv, what=f"dval ({agg})")


def test_gcn_training_reduces_loss():
    g = gen.powerlaw_graph(4000, 80000, gamma=2.4, n_comm=4, mu=0.1, seed=12)
    dg = upload(g)
    op = gnn.SparseOp(dg)
    torch.manual_seed(0)
    F, C = 32, 4
    X = torch.from_numpy(gen.features(60, g.N, F)).to(DEV)
    y = torch.from_numpy(g.comm.astype(np.int64) % C).to(DEV)   # planted communities
    model = gnn.GCN(F, 64, C).to(DEV)
    opt = torch.optim.Adam(model.parameters(), lr=0.01)
    losses = []
    for _ in range(30):
        opt.zero_grad()
        loss = torch.nn.functional.cross_entropy(model(op, X), y)
        loss.backward()
        opt.step()
        losses.append(loss.item())
    assert losses[-1] < 0.7 * losses[0], losses


@pytest.mark.parametrize("seed", range(40))
def test_randomized_configurations(seed):
    """Seeded fuzz over shapes and every plan/kernel knob: random sparsity with empty rows
    and hubs, K (odd/even, > 512), forced chunk / vector width, warps per block, alpha,
    val None, bf16 features, aggregators; every output against the oracle."""
    rng = np.random.default_rng(10_000 + seed)
    M = int(rng.integers(1, 3000))
    N = int(rng.integers(1, 3000))
    nnz = int(rng.integers(0, 40000))
    rows = np.sort(rng.integers(0, M, nnz))
    if nnz > 10 and rng.random() < 0.5:
        rows[: nnz // 3] = rows[0]                       # a hub row
    cols = rng.integers(0, N, nnz)
    vals = rng.uniform(-1, 1, nnz).astype(np.float32)
    g = gen.from_coo(M, N, rows, cols, vals)
    K = int(rng.choice([1, 2, 3, 7, 8, 16, 24, 40, 64, 96, 128, 200, 256, 520, 1024]))
    bf16 = K % 2 == 0 and rng.random() < 0.3
    kw = {}
    if rng.random() < 0.4:
        kw["force_chunk"] = int(rng.choice([1, 3, 8, 17, 32, 64, 100, 128, 256, 512]))
    if rng.random() < 0.3:
        choices = [v for v in ((2, 4, 8, 16) if bf16 else (1, 2, 4, 8)) if K % v == 0]
        if choices:
            kw["force_vw"] = int(rng.choice(choices))
    if rng.random() < 0.3:
        kw["warps_per_block"] = int(rng.choice([1, 2, 4, 16]))
    if rng.random() < 0.3:
        kw["alpha"] = int(rng.choice([1, 3, 8]))
    if rng.random() < 0.2:
        kw["no_locality"] = True
    if rng.random() < 0.2:  # device-parameter overrides, fed to the oracle as well
        kw["num_sms"] = int(rng.integers(1, 300))
        kw["active_blocks_per_sm"] = int(rng.integers(1, 17))
        kw["l2_bytes"] = int(rng.choice([1 << 20, 40 << 20, 126 << 20]))
    with_val = rng.random() < 0.8
    dg = upload(g, with_val=with_val)
    p = gs.plan(dg, K, feature_dtype="bf16" if bf16 else "f32", **kw)
    oracle_plan_checked(p, g, K, feature_dtype="bf16" if bf16 else "f32", **kw)
    X = torch.from_numpy(gen.features(seed, N, K)).to(DEV)
    A1 = torch.from_numpy(gen.features(seed + 1, M, K)).to(DEV)
    if bf16:
        X, A1 = X.to(torch.bfloat16), A1.to(torch.bfloat16)
    Xh, A1h = X.float().cpu().numpy(), A1.float().cpu().numpy()
    val = g.val if with_val else None
    agg = "sum" if bf16 else str(rng.choice(["sum", "sum", "mean", "max", "min"]))
    O = gs.spmm(p, dg, X, agg=agg).cpu().numpy()
    ref, T = oracle.spmm_agg(g.row_ind, g.col_ind, val, Xh, agg, M=M)
    assert_within(O, ref, T, tol=1e-5 if agg in ("sum", "mean") else 1e-6, what=f"spmm {agg}")
    if p.info()["slices"] <= 4:
        E = gs.sddmm(p, dg, A1, X).cpu().numpy()
        r2, T2 = oracle.sddmm(g.row_ind, g.col_ind, val, A1h, Xh)
        assert_within(E, r2, T2, what="sddmm")


@pytest.mark.parametrize("agg", ["sum", "max", "mean"])
@pytest.mark.parametrize("C", [0, 8, 64])
@pytest.mark.parametrize("K", [64, 256])
def test_deterministic_spmm_bitwise_reproducible(agg, C, K):
    """deterministic plans (no atomics: split-row partials summed in chunk order) give the
    same bits on every run, and match the oracle (K = 256: the widened launch shape, rows
    of two vectors per lane run on twice the lanes, writes the per-chunk partials too)."""
    for g in graphs():
        dg = upload(g)
        p = gs.plan(dg, K, force_chunk=C, deterministic=True)
        X = torch.from_numpy(gen.features(70, g.N, K)).to(DEV)
        outs = [gs.spmm(p, dg, X, agg=agg).cpu().numpy() for _ in range(3)]
        assert all(np.array_equal(outs[0], o) for o in outs[1:])
        ref, T = oracle.spmm_agg(g.row_ind, g.col_ind, g.val, X.cpu().numpy(), agg, M=g.M)
        assert_within(outs[0], ref, T, tol=1e-5 if agg != "max" else 1e-6, what=f"det {agg}")
        O = torch.from_numpy(outs[0].copy()).to(DEV)
        if agg == "sum":  # beta = 1 through the fix-up pass as well
            gs.spmm(p, dg, X, out=O, accumulate=True)
            assert_within(O.cpu().numpy(), 2 * ref, 2 * T, what="det accumulate")


# ------------------------------------------------ max / min backward (f3) ---
def _extremum_bounds(g, A, dO):
    """Upper bounds of sum|terms| for dA (N x K) and dval (nnz), independent of which
    term each (row, column) selects: the tolerance scale of the float-atomic sums."""
    v = np.abs(g.val.astype(np.float64)) if g.val is not None else np.ones(g.nnz)
    TdA = np.zeros((g.N, A.shape[1]))
    np.add.at(TdA, g.col_ind, v[:, None] * np.abs(dO[g.row_ind].astype(np.float64)))
    Tdv = (np.abs(A[g.col_ind].astype(np.float64)) * np.abs(dO[g.row_ind])).sum(1)
    return TdA, Tdv


@pytest.mark.parametrize("agg", ["max", "min"])
@pytest.mark.parametrize("K", [1, 7, 32, 100])
@pytest.mark.parametrize("relu", [False, True])
def test_extremum_backward_matches_oracle(agg, K, relu):
    """gnn_spmm_extremum_backward against the oracle's first-occurrence subgradient on
    graphs with empty rows, duplicates and a hub, values of both signs; relu=True zeroes
    half the features so most (row, column) maxima are ties between zeros."""
    for g in graphs():
        dg = upload(g)
        X = gen.features(41 + K, g.N, K)
        if relu:
            X = np.maximum(X, 0)
        dO = gen.features(43 + K, g.M, K)
        Xd = torch.from_numpy(X).to(DEV)
        for C in (0, 8):  # rows split across chunks meet in the float atomics (+-0 included)
            Oc = gs.spmm(gs.plan(dg, K, force_chunk=C), dg, Xd, agg=agg).cpu().numpy()
            rO, TO = oracle.spmm_agg(g.row_ind, g.col_ind, g.val, X, agg, M=g.M)
            assert_within(Oc, rO, TO, what=f"{agg} forward K={K} relu={relu} C={C}")
        p = gs.plan(dg, K)
        O = gs.spmm(p, dg, Xd, agg=agg)
        dval = torch.zeros(g.nnz, device=DEV)
        dA, _ = gs.spmm_extremum_backward(dg, agg, Xd, O, torch.from_numpy(dO).to(DEV),
                                          dval=dval)
        torch.cuda.synchronize()
        rA, rv = oracle.spmm_extremum_backward(g.row_ind, g.col_ind, g.val, X, dO, agg, M=g.M)
        TdA, Tdv = _extremum_bounds(g, X, dO)
        assert_within(dA.cpu().numpy(), rA, TdA, what=f"{agg} dA K={K} relu={relu}")
        assert_within(dval.cpu().numpy(), rv, Tdv, what=f"{agg} dval K={K} relu={relu}")


def test_extremum_backward_matches_torch_scatter_reduce():
    """An independent library reference on tie-free data: torch's scatter_reduce(amax /
    amin) autograd (ties split evenly there; none occur here) gives the same dX and dv."""
    rng = np.random.default_rng(11)
    M, N, K = 300, 400, 16
    rows = np.sort(rng.integers(0, M, 5000))
    cols = rng.integers(0, N, rows.size)
    keep = np.sort(np.unique(rows * N + cols, return_index=True)[1])
    rows, cols = rows[keep], cols[keep]
    g = gen.from_coo(M, N, rows, cols, rng.uniform(0.5, 1.5, rows.size).astype(np.float32))
    dg = upload(g)
    X = torch.randn(N, K, device=DEV, dtype=torch.float64).float().requires_grad_()
    v = torch.from_numpy(g.val).to(DEV).requires_grad_()
    dO = torch.randn(M, K, device=DEV)
    op = gnn.SparseOp(dg)
    ri = torch.from_numpy(g.row_ind.astype(np.int64)).to(DEV)
    ci = torch.from_numpy(g.col_ind.astype(np.int64)).to(DEV)
    present = torch.zeros(M, dtype=torch.bool, device=DEV)
    present[ri] = True
    for agg, red in (("max", "amax"), ("min", "amin")):
        O = gnn.spmm_autograd(op, X, v, agg=agg)
        (O * dO).sum().backward()
        gX, gv = X.grad.clone(), v.grad.clone()
        X.grad = v.grad = None
        terms = v[:, None] * X[ci]
        Oref = torch.zeros(M, K, device=DEV).scatter_reduce(
            0, ri[:, None].expand(-1, K), terms, reduce=red, include_self=False)
        Oref = torch.where(present[:, None], Oref, torch.zeros_like(Oref))
        assert torch.equal(O.detach(), Oref.detach())
        (Oref * dO).sum().backward()
        torch.testing.assert_close(gX, X.grad, rtol=1e-5, atol=1e-5)
        torch.testing.assert_close(gv, v.grad, rtol=1e-5, atol=1e-5)
        X.grad = v.grad = None


@pytest.mark.parametrize("K", [32, 256])
def test_deterministic_bf16_spmm(K):
    """bf16 features through a deterministic plan (widened launch at K = 256): same bits
    on every run, within the fp32 bar of the oracle fed the exact bf16 values."""
    for g in graphs():
        dg = upload(g)
        p = gs.plan(dg, K, deterministic=True, feature_dtype="bf16")
        Xb = torch.from_numpy(gen.features(71, g.N, K)).to(torch.bfloat16).to(DEV)
        outs = [gs.spmm(p, dg, Xb).cpu().numpy() for _ in range(3)]
        assert all(np.array_equal(outs[0], o) for o in outs[1:])
        ref, T = oracle.spmm(g.row_ind, g.col_ind, g.val, Xb.float().cpu().numpy(), M=g.M)
        assert_within(outs[0], ref, T, what=f"det bf16 K={K}")
