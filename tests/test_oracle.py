"""Pins for the CPU oracle (runs without a GPU).

The oracle (oracle/oracle.c) is checked against things other than itself:
dense fp64 brute force, scipy.sparse, closed forms, invariants, the paper's
Fig. 4 / Fig. 5 worked example (tests/golden/fig4_fig5_warp2.txt) and brute-force
enumerations.  A dropped term, wrong sign/index or transposed operand in any
oracle function fails at least one test here.
"""
import os

import numpy as np
import pytest
import scipy.sparse as sp

import gen
import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ----------------------------------------------------------------- helpers --
def random_coo(rng, M, N, nnz, dup=True, empty_rows=True, vals=True):
    """Random hybrid CSR/COO with duplicates and empty rows allowed."""
    rows = rng.integers(0, M, nnz)
    if empty_rows and M > 4:
        rows = np.where(rows % 5 == 3, (rows + 1) % M, rows)  # leave gaps
    cols = rng.integers(0, N, nnz)
    if dup and nnz > 4:
        rows[-2:] = rows[:2]
        cols[-2:] = cols[:2]
    v = rng.uniform(-1, 1, nnz).astype(np.float32) if vals else None
    return gen.from_coo(M, N, rows, cols, v if v is not None else np.ones(nnz, np.float32)), v is None


def dense_of(g, use_val=True):
    S = np.zeros((g.M, g.N), np.float64)
    np.add.at(S, (g.row_ind.astype(np.int64), g.col_ind.astype(np.int64)),
              g.val.astype(np.float64) if use_val else 1.0)
    return S


def load_fig4():
    d = {}
    with open(os.path.join(GOLDEN, "fig4_fig5_warp2.txt")) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, *v = line.split()
            d[k] = v
    entries = [tuple(int(x) for x in e.split(":")) for e in d["entries"]]
    return int(d["nnz_per_warp"][0]), int(d["num_warps"][0]), int(d["K"][0]), \
        int(d["warp"][0]), entries


def fig4_matrix():
    """A 25-nnz, 7x7 matrix consistent with the Fig. 4/5 captions: nnz [10,15) are
    (3,4) (3,5) (3,6) (4,1) (4,2); the rest (lost with the figure) is filler."""
    C, W, K, w, entries = load_fig4()
    rows = [0, 0, 0, 1, 1, 1, 1, 2, 2, 2] + [r for r, _ in entries] + [4, 5, 5, 6, 6, 6, 6, 6, 6, 6][:W * C - 15]
    cols = [0, 2, 5, 1, 2, 3, 6, 0, 4, 6] + [c for _, c in entries] + [3, 0, 5, 0, 1, 2, 3, 4, 5, 6][:W * C - 15]
    return gen.from_coo(7, 7, rows, cols), C, K, w, entries


# -------------------------------------------------------------------- SpMM --
@pytest.mark.parametrize("seed", range(6))
def test_spmm_matches_dense_bruteforce(seed):
    rng = np.random.default_rng(seed)
    M, N, K = int(rng.integers(1, 60)), int(rng.integers(1, 60)), int(rng.integers(1, 40))
    g, _ = random_coo(rng, M, N, int(rng.integers(0, 400)))
    A = rng.uniform(-1, 1, (N, K)).astype(np.float32)
    O, T = oracle.spmm(g.row_ind, g.col_ind, g.val, A, M=M)
    S = dense_of(g)
    ref = S @ A.astype(np.float64)
    np.testing.assert_allclose(O, ref, rtol=0, atol=1e-12)
    # T is the sum of |terms| (duplicates contribute one term each)
    Tref = np.zeros((M, K))
    np.add.at(Tref, g.row_ind, np.abs(g.val[:, None].astype(np.float64) * A[g.col_ind].astype(np.float64)))
    np.testing.assert_allclose(T, Tref, rtol=1e-12, atol=0)


def test_spmm_val_none_is_ones():
    rng = np.random.default_rng(11)
    g, _ = random_coo(rng, 30, 20, 200)
    A = rng.uniform(-1, 1, (20, 8)).astype(np.float32)
    O, _ = oracle.spmm(g.row_ind, g.col_ind, None, A, M=30)
    np.testing.assert_allclose(O, dense_of(g, use_val=False) @ A.astype(np.float64), atol=1e-12)


def test_spmm_matches_scipy_on_generated_graph():
    g = gen.powerlaw_graph(3000, 30000, gamma=2.5, n_comm=5, seed=21)
    A = gen.features(5, g.N, 24)
    O, _ = oracle.spmm(g.row_ind, g.col_ind, g.val, A, M=g.M)
    S = sp.csr_matrix((g.val.astype(np.float64), g.col_ind, g.row_ptr), shape=(g.M, g.N))
    np.testing.assert_allclose(O, S @ A.astype(np.float64), rtol=0, atol=1e-12)


def test_spmm_identity_returns_A_exactly():
    N, K = 50, 16
    A = gen.features(1, N, K)
    O, _ = oracle.spmm(np.arange(N), np.arange(N), np.ones(N, np.float32), A, M=N)
    assert np.array_equal(O, A.astype(np.float64))


def test_spmm_ones_features_give_row_value_sums():
    rng = np.random.default_rng(3)
    M, N, K = 40, 30, 5
    g, _ = random_coo(rng, M, N, 300)
    v = rng.integers(1, 5, g.nnz).astype(np.float32)
    O, _ = oracle.spmm(g.row_ind, g.col_ind, v, np.ones((N, K), np.float32), M=M)
    sums = np.bincount(g.row_ind, weights=v.astype(np.float64), minlength=M)
    assert np.array_equal(O, np.repeat(sums[:, None], K, 1))


def test_spmm_all_ones_row_gives_column_sums():
    N, K = 37, 9
    A = gen.features(2, N, K)
    O, _ = oracle.spmm(np.zeros(N, np.int32), np.arange(N), None, A, M=1)
    np.testing.assert_allclose(O[0], A.astype(np.float64).sum(0), atol=1e-13)


def test_spmm_duplicate_edge_doubles():
    A = gen.features(3, 4, 6)
    O1, _ = oracle.spmm([0], [2], np.float32([0.75]), A, M=1)
    O2, _ = oracle.spmm([0, 0], [2, 2], np.float32([0.75, 0.75]), A, M=1)
    assert np.array_equal(O2, 2 * O1)


def test_spmm_power_of_two_scaling_exact():
    rng = np.random.default_rng(4)
    g, _ = random_coo(rng, 25, 25, 150)
    A = gen.features(4, 25, 7)
    O, _ = oracle.spmm(g.row_ind, g.col_ind, g.val, A, M=25)
    O8, _ = oracle.spmm(g.row_ind, g.col_ind, g.val, A * np.float32(8), M=25)
    assert np.array_equal(O8, 8 * O)


def test_spmm_permutation_equivariance():
    g = gen.powerlaw_graph(500, 5000, gamma=2.5, n_comm=3, seed=9)
    A = gen.features(9, g.N, 12)
    perm = np.random.default_rng(0).permutation(g.N)  # new id of node i
    gp = gen.from_coo(g.M, g.N, perm[g.row_ind], perm[g.col_ind], g.val)
    Ap = np.empty_like(A)
    Ap[perm] = A
    O, _ = oracle.spmm(g.row_ind, g.col_ind, g.val, A, M=g.M)
    Op, _ = oracle.spmm(gp.row_ind, gp.col_ind, gp.val, Ap, M=g.M)
    np.testing.assert_allclose(Op[perm], O, atol=1e-12)


def test_spmm_row_range_and_rows_sample_agree_with_full():
    g = gen.powerlaw_graph(800, 8000, gamma=2.4, n_comm=4, seed=10)
    A = gen.features(10, g.N, 8)
    O, T = oracle.spmm(g.row_ind, g.col_ind, g.val, A, M=g.M)
    rows = np.array([0, 5, 799, 400])
    Os, Ts = oracle.spmm_rows(g, A, rows)
    assert np.array_equal(Os, O[rows]) and np.array_equal(Ts, T[rows])
    with pytest.raises(ValueError):  # a row outside the window is a contract error
        oracle.spmm(g.row_ind, g.col_ind, g.val, A, i0=0, i1=g.nnz, r0=1, nrows=10)


def test_spmm_fig4_worked_example():
    g, C, K, w, entries = fig4_matrix()
    A = gen.features(12, 7, K)
    O, _ = oracle.spmm(g.row_ind, g.col_ind, g.val, A, M=7, i0=w * C, i1=(w + 1) * C,
                       r0=0, nrows=7)
    # warp 2 writes A4+A5+A6 into O row 3 and A1+A2 into O row 4
    A64 = A.astype(np.float64)
    np.testing.assert_allclose(O[3], A64[4] + A64[5] + A64[6], atol=1e-15)
    np.testing.assert_allclose(O[4], A64[1] + A64[2], atol=1e-15)
    assert not O[[0, 1, 2, 5, 6]].any()


# ------------------------------------------------------------------- SDDMM --
@pytest.mark.parametrize("seed", range(6))
def test_sddmm_matches_dense_bruteforce(seed):
    rng = np.random.default_rng(100 + seed)
    M, N, K = int(rng.integers(1, 50)), int(rng.integers(1, 50)), int(rng.integers(1, 40))
    g, _ = random_coo(rng, M, N, int(rng.integers(0, 300)))
    A1 = rng.uniform(-1, 1, (M, K)).astype(np.float32)
    A2 = rng.uniform(-1, 1, (K, N)).astype(np.float32)       # Table I: A2 is K x N
    A2T = np.ascontiguousarray(A2.T)
    out, T = oracle.sddmm(g.row_ind, g.col_ind, g.val, A1, A2T)
    D = A1.astype(np.float64) @ A2.astype(np.float64)        # (A1 A2)
    ref = D[g.row_ind, g.col_ind] * g.val.astype(np.float64)  # (.) S at the nonzeros
    np.testing.assert_allclose(out, ref, rtol=0, atol=1e-12)
    Tref = (np.abs(A1.astype(np.float64)) @ np.abs(A2.astype(np.float64)))[g.row_ind, g.col_ind] \
        * np.abs(g.val.astype(np.float64))
    np.testing.assert_allclose(T, Tref, rtol=1e-12, atol=1e-300)


def test_sddmm_self_loop_is_squared_norm():
    X = gen.features(20, 30, 33)
    out, _ = oracle.sddmm(np.arange(30), np.arange(30), None, X, X)
    np.testing.assert_allclose(out, (X.astype(np.float64) ** 2).sum(1), rtol=1e-15)


def test_sddmm_ones_give_v_times_K():
    v = np.float32([0.5, 2.0, 3.0, 1.0])
    out, _ = oracle.sddmm([0, 0, 1, 2], [1, 2, 0, 2], v, np.ones((3, 17), np.float32),
                          np.ones((3, 17), np.float32))
    assert np.array_equal(out, v.astype(np.float64) * 17)


def test_sddmm_pair_symmetry_bitwise():
    X = gen.features(21, 10, 19)
    out, _ = oracle.sddmm([2, 7], [7, 2], None, X, X)
    assert out[0] == out[1]


def test_sddmm_scale_applied_after_sum():
    # S_O[i] <- S_O[i] * v (Algo 2 line 6): negative v flips the sign exactly
    X = gen.features(22, 4, 8)
    a, _ = oracle.sddmm([0], [3], np.float32([1.0]), X, X)
    b, _ = oracle.sddmm([0], [3], np.float32([-0.25]), X, X)
    assert b[0] == -0.25 * a[0]


def test_spmm_sddmm_adjoint_identity():
    """sum_{r,k} G[r,k] SpMM(S,X)[r,k] == sum_i SDDMM(G, X; S)[i]
    (SDDMM is the gradient of SpMM w.r.t. the edge values)."""
    g = gen.powerlaw_graph(600, 6000, gamma=2.4, n_comm=3, seed=23)
    X = gen.features(23, g.N, 16)
    G = gen.features(24, g.M, 16)
    O, _ = oracle.spmm(g.row_ind, g.col_ind, g.val, X, M=g.M)
    out, T = oracle.sddmm(g.row_ind, g.col_ind, g.val, G, X)
    lhs = float((G.astype(np.float64) * O).sum())
    rhs = float(out.sum())
    assert abs(lhs - rhs) <= 1e-12 * float(T.sum())


def test_sddmm_fig5_worked_example():
    g, C, K, w, entries = fig4_matrix()
    X1 = gen.features(30, 7, K)
    X2 = gen.features(31, 7, K)
    out, _ = oracle.sddmm(g.row_ind, g.col_ind, g.val, X1, X2, i0=w * C, i1=(w + 1) * C)
    # first output of warp 2 is S_O(3, 4) = <A1 row 3, A2 column 4>
    for j, (r, c) in enumerate(entries):
        ref = float(np.dot(X1[r].astype(np.float64), X2[c].astype(np.float64)))
        assert abs(out[j] - ref) <= 1e-15


# -------------------------------------------------------------------- plan --
def _brute_blocks(nnz, C, S, G, WPB):
    """Enumerate work items (chunk, slice) -> lane group -> warp -> block."""
    nch = -(-nnz // C) if nnz else 0
    items = np.arange(nch * S)
    groups_ = items                      # one lane group per work item
    warps = groups_ // G
    blocks = warps // WPB
    return int(np.unique(blocks).size)


VW_TABLE = {  # K: (vw_feat, lanes, vecs, slices, groups) -- DESIGN.md "Plan rule" table
    32: (8, 4, 1, 1, 8), 64: (8, 8, 1, 1, 4), 128: (8, 8, 2, 1, 4), 256: (8, 16, 2, 1, 2),
    100: (4, 16, 2, 1, 2), 33: (1, 32, 2, 1, 1), 1000: (8, 32, 2, 2, 1), 6: (2, 4, 1, 1, 8),
    1: (1, 1, 1, 1, 32), 512: (8, 32, 2, 1, 1), 24: (8, 4, 1, 1, 8), 12: (4, 4, 1, 1, 8),
    2048: (8, 32, 2, 4, 1), 120: (8, 16, 1, 1, 2),
}


@pytest.mark.parametrize("K", sorted(VW_TABLE))
def test_plan_vector_width_table(K):
    p = oracle.plan(np.zeros(100, np.int32), K, num_sms=148, active_blocks_per_sm=8)
    assert (p.info["vw_feat"], p.info["lanes"], p.info["vecs"], p.info["slices"],
            p.info["groups"]) == VW_TABLE[K]


@pytest.mark.parametrize("nnz,K,alpha,abs_", [
    (0, 32, 2, 8), (1, 32, 2, 8), (10_000, 32, 2, 8), (100_000, 64, 2, 8),
    (1_500_000, 128, 2, 8), (5_000_000, 32, 2, 4), (3_000_000, 256, 1, 6),
    (20_000_000, 64, 4, 8), (123_457, 100, 2, 3)])
def test_plan_dtp_maximality_bruteforce(nnz, K, alpha, abs_):
    nsm, wpb = 148, 8
    p = oracle.plan(np.zeros(nnz, np.int32), K, num_sms=nsm, active_blocks_per_sm=abs_,
                    alpha=alpha, warps_per_block=wpb)
    S, G, C = p.info["slices"], p.info["groups"], p.info["chunk"]
    need = alpha * nsm * abs_
    cands = [8, 32, 64, 128, 256, 512]
    ok = [c for c in cands if _brute_blocks(nnz, c, S, G, wpb) >= need]
    assert C == (max(ok) if ok else 8)
    assert p.info["num_blocks"] == (_brute_blocks(nnz, C, S, G, wpb) if nnz else 0)
    assert p.info["num_chunks"] == (-(-nnz // C) if nnz else 0)
    assert p.info["vw_sparse"] == {8: 1, 32: 1, 64: 2, 128: 4, 256: 4, 512: 4}[C]


# ---- step 5b, the locality cap: hand-worked examples ----
# 148 SMs x 2 blocks/SM -> FW = 296; WPB 8; K = 256 fp32 -> L 16, R 2, G 2, S 1.
# nnz = 10,000,000, M = 200,000 (degree 50): DTP alone -> 512 (blocks(512) = 1221 >= 592).
# L2 = 64 MiB: rows that fit = (67,108,864 / 4) / (256 * 4) = 16,384.
#   C = 512: 296*8*2*512 = 2,424,832 nnz in flight * 200,000 / 10^7 = 48,496 rows  > 16,384
#   C = 256: 1,212,416 -> 24,248 rows > 16,384;  C = 128: 606,208 -> 12,124 rows <= 16,384
# bf16: VW 16 -> L 8, R 2, G 4 (twice the chunks in flight) and 2 B per element (twice
#   the rows fit, 32,768): C = 256 -> 48,496 rows > 32,768; C = 128 -> 24,248 -> 128.
# Degree 100 (M = 100,000), fp32: C = 512 -> 24,248 > 16,384; C = 256 -> 12,124 -> 256.
# Degree 500 (M = 20,000): C = 512 -> 4,849 rows -> 512.  L2 off -> 512.
# L2 = 1 MiB: 256 rows fit; even C = 8 (37,888 nnz -> 757 rows) does not -> 8.  The
# step-5c chunk floor does NOT raise it: it applies only where InEq. (5) itself chose
# fewer than 64 (here C_dtp = 512; the cap, not a lack of parallelism, decided).
@pytest.mark.parametrize("M,dtype,l2,expect", [
    (200_000, 0, 64 << 20, 128), (200_000, 1, 64 << 20, 128), (100_000, 0, 64 << 20, 256),
    (200_000, 0, 0, 512), (20_000, 0, 64 << 20, 512), (200_000, 0, 1 << 20, 8)])
def test_plan_locality_cap_worked_examples(M, dtype, l2, expect):
    p = oracle.plan(np.zeros(10_000_000, np.int32), 256, num_sms=148, active_blocks_per_sm=2,
                    feature_dtype=dtype, M=M, l2_bytes=l2)
    assert p.info["chunk_dtp"] == 512
    assert p.info["chunk"] == expect
    assert p.info["num_chunks"] == -(-10_000_000 // expect)


def test_plan_locality_cap_monotone():
    """More L2 never shrinks C*, more rows per nonzero never grows it, the cap never
    exceeds the DTP choice, an unbounded L2 gives DTP exactly, and where DTP itself chose
    8 or 32 the step-5c floor gives 64 whatever the L2 (no L2 model: DTP exactly)."""
    rng = np.random.default_rng(77)
    cands = [8, 32, 64, 128, 256, 512]
    for _ in range(60):
        nnz = int(rng.integers(1, 3_000_000))
        K = int(rng.choice([8, 32, 64, 128, 256, 512, 1024]))
        abs_ = int(rng.integers(1, 9))
        dt = int(rng.integers(0, 2)) if K % 2 == 0 else 0
        row_ind = np.zeros(nnz, np.int32)

        def chunk(M, l2):
            return oracle.plan(row_ind, K, 148, abs_, feature_dtype=dt, M=M,
                               l2_bytes=l2).info

        M = int(rng.integers(1, 2 * nnz + 2))
        base = chunk(M, 0)
        assert base["chunk"] == base["chunk_dtp"]
        prev = 0
        for l2 in (1 << 16, 1 << 20, 16 << 20, 64 << 20, 126 << 20, 1 << 40):
            c = chunk(M, l2)["chunk"]
            if base["chunk"] < 64:
                assert c == 64
            else:
                assert c in cands and c <= base["chunk"] and c >= prev
            prev = c
        assert prev == max(base["chunk"], 64)
        c_small_m = chunk(max(1, M // 4), 64 << 20)["chunk"]
        assert c_small_m >= chunk(M, 64 << 20)["chunk"]


def test_plan_matches_survey_dtp_table():
    """SURVEY.md §8(a1) table (WPB 8, 8 blocks/SM, 148 SMs, alpha 2)."""
    for nnz, K, C in [(10_000, 32, 8), (100_000, 64, 8), (114_848_857, 32, 512),
                      (114_848_857, 256, 512), (126_167_053, 256, 512)]:
        assert oracle.plan(np.zeros(1, np.int32), K, 148, 8).info  # smoke
        p = oracle.plan(np.zeros(nnz, np.int32), K, 148, 8)
        assert p.info["chunk"] == C, (nnz, K)


@pytest.mark.parametrize("seed", range(4))
def test_plan_chunk_arrays_against_csr_scan(seed):
    rng = np.random.default_rng(200 + seed)
    g, _ = random_coo(rng, int(rng.integers(1, 300)), 50, int(rng.integers(1, 3000)))
    C = int(rng.choice([1, 3, 5, 8, 32, 64, 128]))
    p = oracle.plan(g.row_ind, 32, 148, 8, force_chunk=C)
    nnz = g.nnz
    assert p.info["chunk"] == C and p.info["num_chunks"] == -(-nnz // C)
    for c in range(p.info["num_chunks"]):
        s, e = c * C, min(c * C + C, nnz)
        rf, rl = p.row_first[c], p.row_last[c]
        # row_first is the row owning nnz s: row_ptr[rf] <= s < row_ptr[rf+1]
        assert g.row_ptr[rf] <= s < g.row_ptr[rf + 1]
        assert g.row_ptr[rl] <= e - 1 < g.row_ptr[rl + 1]
        head = g.row_ptr[rf] < s                 # row rf has nnz before this chunk
        tail = g.row_ptr[rl + 1] > e             # row rl has nnz after this chunk
        assert p.flags[c] == (int(head) | (int(tail) << 1))


def test_plan_fig4_forced_chunk_5():
    g, C, K, w, entries = fig4_matrix()
    p = oracle.plan(g.row_ind, K, 148, 8, force_chunk=C)
    assert p.info["num_chunks"] == 5
    assert p.row_first[w] == entries[0][0] == 3
    assert p.row_last[w] == entries[-1][0] == 4
    # the row switch happens inside the chunk: nnz 12 is row 3, nnz 13 row 4
    assert g.row_ind[w * C + 2] == 3 and g.row_ind[w * C + 3] == 4


def test_plan_rejects_bad_args():
    with pytest.raises(ValueError):
        oracle.plan(np.zeros(4, np.int32), 0, 148, 8)
    with pytest.raises(ValueError):
        oracle.plan(np.zeros(4, np.int32), 30, 148, 8, force_vw=4)


# ------------------------------------------------------------------ shards --
@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_shard_rows_bruteforce(P):
    g = gen.powerlaw_graph(2000, 40000, gamma=2.2, n_comm=4, seed=40)
    b = oracle.shard_rows(g.row_ptr, P)
    nnz = g.nnz
    assert b[0] == 0 and b[P] == g.M and (np.diff(b) >= 0).all()
    for p in range(1, P):
        t = p * nnz // P
        brute = next(r for r in range(g.M + 1) if g.row_ptr[r] >= t)
        assert b[p] == brute
    maxdeg = int(np.diff(g.row_ptr).max())
    for p in range(P):
        share = int(g.row_ptr[b[p + 1]] - g.row_ptr[b[p]])
        assert abs(share - nnz / P) <= maxdeg + 1


def test_shard_rows_subview_and_empty_shards():
    row_ptr = np.array([100, 100, 100, 130, 130], np.int32)  # sub-view, one heavy row
    b = oracle.shard_rows(row_ptr, 4)
    assert list(b) == [0, 3, 3, 3, 4]
    assert b[0] == 0 and b[-1] == 4


@pytest.mark.parametrize("nnz,P", [(0, 4), (10, 3), (114_848_857, 8), (7, 8)])
def test_shard_edges(nnz, P):
    b = oracle.shard_edges(nnz, P)
    assert b[0] == 0 and b[-1] == nnz and (np.diff(b) >= 0).all()
    assert (np.diff(b) <= -(-nnz // P)).all()


# Hand-worked floor(p * nnz / P) bounds (SURVEY §8(c) "Shards"), chosen where
# floor and ceil (and rounding) give different answers: 10/3 = 3.33 -> 3, 20/3 = 6.67 -> 6
# (ceil would give [0, 4, 7, 10], rounding [0, 3, 7, 10]); 7 edges over 8 ranks leave
# rank 0 empty (floor(7/8) = 0) and rank 7 holds one edge (floor(49/8) = 6).
@pytest.mark.parametrize("nnz,P,expect", [
    (10, 3, [0, 3, 6, 10]),
    (7, 8, [0, 0, 1, 2, 3, 4, 5, 6, 7]),
    (11, 4, [0, 2, 5, 8, 11]),
    (5, 2, [0, 2, 5]),
    (1, 3, [0, 0, 0, 1]),
    (0, 2, [0, 0, 0]),
])
def test_shard_edges_hand_worked(nnz, P, expect):
    assert list(oracle.shard_edges(nnz, P)) == expect


def test_shard_edges_no_int64_overflow_at_full_scale():
    # p * nnz exceeds 2^31 at C4/C5 sizes; the bound must still be the exact floor
    nnz, P = 126_167_053, 8
    b = oracle.shard_edges(nnz, P)
    assert list(b) == [p * nnz // P for p in range(P + 1)]
    assert b[5] == 78_854_408  # 5 * 126,167,053 / 8 = 78,854,408.125


def test_assert_within_rejects_nan_and_inf():
    from helpers import assert_within
    ref = np.array([1.0, 2.0]); T = np.array([1.0, 2.0])
    assert assert_within(np.array([1.0, 2.0]), ref, T) == 0.0
    for bad in (np.nan, np.inf, -np.inf):
        with pytest.raises(AssertionError):
            assert_within(np.array([1.0, bad]), ref, T)
    with pytest.raises(AssertionError):  # a NaN where sum|terms| == 0 fails too
        assert_within(np.array([np.nan]), np.array([0.0]), np.array([0.0]))


def test_csr_to_coo_matches_repeat():
    g = gen.powerlaw_graph(300, 3000, seed=41)
    assert np.array_equal(oracle.csr_to_coo(g.row_ptr), g.row_ind)
    assert np.array_equal(np.repeat(np.arange(g.M), np.diff(g.row_ptr)), g.row_ind)


BF16_TABLE = {  # K: (vw_feat, lanes, vecs, slices, groups) with bf16 features
    32: (16, 2, 1, 1, 16), 64: (16, 4, 1, 1, 8), 128: (16, 8, 1, 1, 4), 256: (16, 8, 2, 1, 4),
    24: (8, 4, 1, 1, 8), 6: (2, 4, 1, 1, 8), 512: (16, 16, 2, 1, 2), 1000: (8, 32, 2, 2, 1),
}


@pytest.mark.parametrize("K", sorted(BF16_TABLE))
def test_plan_bf16_vector_width_table(K):
    p = oracle.plan(np.zeros(100, np.int32), K, 148, 8, feature_dtype=1)
    assert (p.info["vw_feat"], p.info["lanes"], p.info["vecs"], p.info["slices"],
            p.info["groups"]) == BF16_TABLE[K]
    assert p.info["feature_dtype"] == 1


def test_plan_bf16_rejects_odd_K_and_bad_force_vw():
    with pytest.raises(ValueError):
        oracle.plan(np.zeros(10, np.int32), 33, 148, 8, feature_dtype=1)
    with pytest.raises(ValueError):
        oracle.plan(np.zeros(10, np.int32), 32, 148, 8, feature_dtype=1, force_vw=1)
    with pytest.raises(ValueError):
        oracle.plan(np.zeros(10, np.int32), 32, 148, 8, feature_dtype=0, force_vw=16)


# ------------------------------------------------------ aggregators (f3) ----
@pytest.mark.parametrize("agg", ["sum", "mean", "max", "min"])
@pytest.mark.parametrize("seed", range(3))
def test_spmm_aggregators_match_numpy_definition(agg, seed):
    """Eq. 1 with (+) in {sum, mean, max, min} against a per-row numpy reduction over the
    row's term matrix (empty rows -> 0)."""
    rng = np.random.default_rng(300 + seed)
    M, N, K = 40, 30, 7
    g, _ = random_coo(rng, M, N, 400)
    A = rng.uniform(-1, 1, (N, K)).astype(np.float32)
    O, T = oracle.spmm_agg(g.row_ind, g.col_ind, g.val, A, agg, M=M)
    terms = g.val[:, None].astype(np.float64) * A[g.col_ind].astype(np.float64)
    for r in range(M):
        tr = terms[g.row_ind == r]
        if tr.shape[0] == 0:
            assert not O[r].any()
            continue
        ref = {"sum": tr.sum(0), "mean": tr.mean(0), "max": tr.max(0), "min": tr.min(0)}[agg]
        np.testing.assert_allclose(O[r], ref, rtol=0, atol=1e-13)
        tref = np.abs(tr).sum(0) / (tr.shape[0] if agg == "mean" else 1) if agg in ("sum", "mean") \
            else np.abs(tr).max(0)
        np.testing.assert_allclose(T[r], tref, rtol=1e-13, atol=0)


def test_spmm_agg_sum_is_algorithm_1():
    rng = np.random.default_rng(9)
    g, _ = random_coo(rng, 30, 20, 200)
    A = rng.uniform(-1, 1, (20, 5)).astype(np.float32)
    a = oracle.spmm_agg(g.row_ind, g.col_ind, g.val, A, "sum", M=30)
    b = oracle.spmm(g.row_ind, g.col_ind, g.val, A, M=30)
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])


# ---------------------------------------------- max / min backward (f3) ----
@pytest.mark.parametrize("agg", ["max", "min"])
@pytest.mark.parametrize("seed", range(3))
def test_extremum_backward_matches_finite_differences(agg, seed):
    """d/dA and d/dval of L = sum(dO * O), O = the max / min aggregation, by central
    differences of the oracle's FORWARD (oracle.spmm_agg, fp64) on tie-free inputs: the
    selected term moves with its inputs, the others do not move O at all."""
    rng = np.random.default_rng(900 + seed)
    M, N, K, nnz = 6, 9, 3, 30
    rows = np.sort(rng.integers(0, M, nnz))
    cols = rng.integers(0, N, nnz)
    keep = np.unique(rows * N + cols, return_index=True)[1]  # no duplicate (r, c): no ties
    rows, cols = rows[np.sort(keep)], cols[np.sort(keep)]
    val = rng.uniform(0.5, 1.5, rows.size).astype(np.float32)
    A = rng.uniform(-1, 1, (N, K)).astype(np.float32)
    dO = rng.uniform(-1, 1, (M, K)).astype(np.float32)
    dA, dval = oracle.spmm_extremum_backward(rows, cols, val, A, dO, agg, M=M)

    def loss(A_, v_):
        O, _ = oracle.spmm_agg(rows, cols, v_, A_, agg, M=M)
        return float((O * dO.astype(np.float64)).sum())

    eps = 2.0 ** -12  # far below the gaps between competing terms (checked below)
    fd_A = np.zeros_like(dA)
    for c in range(N):
        for k in range(K):
            Ap, Am = A.copy(), A.copy()
            Ap[c, k] += eps
            Am[c, k] -= eps
            fd_A[c, k] = (loss(Ap, val) - loss(Am, val)) / (2 * eps)
    fd_v = np.zeros_like(dval)
    for i in range(rows.size):
        vp, vm = val.copy(), val.copy()
        vp[i] += eps
        vm[i] -= eps
        fd_v[i] = (loss(A, vp) - loss(A, vm)) / (2 * eps)
    terms = val[:, None].astype(np.float64) * A[cols]
    for r in range(M):  # tie-free by a margin larger than the perturbation
        t = np.sort(terms[rows == r], axis=0)
        if t.shape[0] > 1:
            assert (np.diff(t, axis=0) > 4 * eps).all()
    np.testing.assert_allclose(dA, fd_A, rtol=0, atol=1e-6)
    np.testing.assert_allclose(dval, fd_v, rtol=0, atol=1e-6)


def test_extremum_backward_ties_go_to_the_first_term():
    """Hand-worked: row 0 has three terms, two of them tied for the max (A[1] = A[2] = 2
    with v = 1) and one tied zero pair in column 1; row 1 is a single term; row 2 empty.
    The first tied nonzero in storage order takes the whole gradient."""
    rows = np.array([0, 0, 0, 1])
    cols = np.array([0, 1, 2, 0])
    val = np.ones(4, np.float32)
    A = np.array([[1.0, 0.0], [2.0, 0.0], [2.0, -1.0]], np.float32)
    dO = np.array([[10.0, 20.0], [30.0, 40.0], [50.0, 60.0]], np.float32)
    dA, dval = oracle.spmm_extremum_backward(rows, cols, val, A, dO, "max", M=3)
    # row 0, col 0: max 2 at nonzeros 1 and 2 -> nonzero 1 (source 1); col 1: max 0 at
    # nonzeros 0 and 1 -> nonzero 0 (source 0).  row 1: nonzero 3 (source 0) everywhere.
    np.testing.assert_array_equal(dA, [[30.0, 20.0 + 40.0], [10.0, 0.0], [0.0, 0.0]])
    np.testing.assert_array_equal(dval, [0.0 * 20.0, 2.0 * 10.0, 0.0, 1.0 * 30.0 + 0.0 * 40.0])
    dA, dval = oracle.spmm_extremum_backward(rows, cols, val, A, dO, "min", M=3)
    # min: col 0 -> nonzero 0 (value 1); col 1 -> nonzero 2 (value -1)
    np.testing.assert_array_equal(dA, [[10.0 + 30.0, 40.0], [0.0, 0.0], [0.0, 20.0]])
    np.testing.assert_array_equal(dval, [10.0, 0.0, -20.0, 30.0])


def test_parallel_oracle_is_bitwise_serial():
    """OpenMP changes no sum's order: SpMM (whole rows per thread, cuts moved to row
    starts, incl. a hub row longer than a thread's share) and SDDMM give identical bits
    with 1 and with many threads."""
    g = gen.powerlaw_graph(3000, 200_000, gamma=2.1, n_comm=5, seed=91)
    ri = g.row_ind.copy()
    ri[: g.nnz // 3] = 0  # a hub spanning several threads' ranges
    ri.sort()
    X = gen.features(92, g.N, 24)
    nmax = oracle.threads()
    try:
        res = []
        for n in (1, 3, max(4, nmax)):
            oracle.threads(n)
            O, T = oracle.spmm(ri, g.col_ind, g.val, X, M=g.M)
            E, T2 = oracle.sddmm(ri, g.col_ind, g.val, X, X)
            res.append((O, T, E, T2))
        for r in res[1:]:
            for a, b in zip(res[0], r):
                assert np.array_equal(a, b)
    finally:
        oracle.threads(nmax)
