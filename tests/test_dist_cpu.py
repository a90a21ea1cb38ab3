"""Multi-process (gloo, world size 2) tests of the multi-GPU host logic on CPU:
shard bounds agree across ranks and with the oracle, the X all-gather reassembles X,
and per-rank shard results (computed here with the oracle, since kernels need a GPU)
concatenate to the unsharded result."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    import gen
    import oracle
    from paper_conf_ipps_fanwc23_b200 import dist as gdist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        g = gen.powerlaw_graph(3001, 60000, gamma=2.2, n_comm=5, seed=90)
        K = 24
        s = gdist.shard_spec(g.row_ptr, g.N, rank, world)
        # all ranks agree on the bounds
        t = torch.tensor([s.r0, s.r1, s.e0, s.e1, s.f0, s.f1], dtype=torch.int64)
        allb = [torch.zeros_like(t) for _ in range(world)]
        dist.all_gather(allb, t)
        # X all-gather: each rank regenerates only its block
        own = torch.from_numpy(gen.features(91, s.x1 - s.x0, K, row0=s.x0))
        Xg = gdist.gather_features(own, s, g.N)[:g.N].numpy()
        X = gen.features(91, g.N, K)
        ok_x = bool(np.array_equal(Xg, X))
        # per-rank SpMM rows and SDDMM edges, gathered back
        O, _ = oracle.spmm(g.row_ind, g.col_ind, g.val, Xg, i0=s.e0, i1=s.e1, r0=s.r0,
                           nrows=s.r1 - s.r0)
        E, _ = oracle.sddmm(g.row_ind, g.col_ind, g.val, Xg, Xg, i0=s.f0, i1=s.f1)
        rows = [None] * world
        edges = [None] * world
        dist.all_gather_object(rows, (s.r0, O))
        dist.all_gather_object(edges, (s.f0, E))
        if rank == 0:
            Ofull, _ = oracle.spmm(g.row_ind, g.col_ind, g.val, X, M=g.M)
            Efull, _ = oracle.sddmm(g.row_ind, g.col_ind, g.val, X, X)
            Ocat = np.concatenate([o for _, o in sorted(rows, key=lambda x: x[0])])
            Ecat = np.concatenate([e for _, e in sorted(edges, key=lambda x: x[0])])
            bounds = [b.tolist() for b in allb]
            ref_rows = oracle.shard_rows(g.row_ptr, world)
            ok_b = all(bounds[p][0] == ref_rows[p] and bounds[p][1] == ref_rows[p + 1]
                       for p in range(world))
            ok_b &= bounds[0][0] == 0 and bounds[-1][1] == g.M
            ok_b &= all(bounds[p][1] == bounds[p + 1][0] for p in range(world - 1))
            q.put((ok_x, ok_b, bool(np.array_equal(Ocat, Ofull)),
                   bool(np.array_equal(Ecat, Efull))))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_gloo_sharding_and_allgather(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=240)
        assert p.exitcode == 0
    ok_x, ok_b, ok_o, ok_e = q.get(timeout=10)
    assert ok_x, "all-gathered X differs from X"
    assert ok_b, "shard bounds disagree"
    assert ok_o, "concatenated row-shard SpMM differs from unsharded"
    assert ok_e, "concatenated edge-shard SDDMM differs from unsharded"


def test_shard_spec_covers_everything():
    import gen
    from paper_conf_ipps_fanwc23_b200 import dist as gdist
    g = gen.powerlaw_graph(1000, 20000, seed=92)
    for world in (1, 2, 3, 8):
        specs = [gdist.shard_spec(g.row_ptr, g.N, r, world) for r in range(world)]
        assert specs[0].r0 == 0 and specs[-1].r1 == g.M
        assert specs[0].f0 == 0 and specs[-1].f1 == g.nnz
        assert sum(s.e1 - s.e0 for s in specs) == g.nnz
        assert sum(s.x1 - s.x0 for s in specs) == g.N
        for a, b in zip(specs, specs[1:]):
            assert a.r1 == b.r0 and a.f1 == b.f0 and a.e1 == b.e0


def _overlap_worker(rank, world, port, q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    import gen
    import oracle
    import paper_conf_ipps_fanwc23_b200 as gs
    from paper_conf_ipps_fanwc23_b200 import dist as gdist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        g = gen.powerlaw_graph(2501, 50000, gamma=2.2, n_comm=5, seed=93)
        K = 16
        s = gdist.shard_spec(g.row_ptr, g.N, rank, world)
        X = gen.features(94, g.N, K)
        Xf = torch.zeros((s.xblk * world, K))
        own = torch.from_numpy(gen.features(94, s.x1 - s.x0, K, row0=s.x0))
        Xf[s.x0:s.x1] = own
        works = gdist.start_block_broadcasts(Xf, s)
        ro, co, vo, b = gs.split_col_blocks(g.row_ind[s.e0:s.e1], g.col_ind[s.e0:s.e1],
                                            g.val[s.e0:s.e1], world, s.xblk)
        O = np.zeros((s.r1 - s.r0, K))
        for qq in gdist.block_order(world, rank):
            if qq != rank:
                works[qq].wait()
            a, z = int(b[qq]), int(b[qq + 1])
            part, _ = oracle.spmm(ro, co, vo, Xf.numpy(), i0=a, i1=z, r0=s.r0,
                                  nrows=s.r1 - s.r0)
            O += part
        ref, _ = oracle.spmm(g.row_ind, g.col_ind, g.val, X, i0=s.e0, i1=s.e1, r0=s.r0,
                             nrows=s.r1 - s.r0)
        ok = bool(np.allclose(O, ref, rtol=0, atol=1e-12)) and bool(
            np.array_equal(Xf[:g.N].numpy(), X))
        res = [None] * world
        dist.all_gather_object(res, ok)
        if rank == 0:
            q.put(all(res))
    finally:
        dist.destroy_process_group()


def test_gloo_overlapped_block_broadcast_spmm():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    world = 2
    procs = [ctx.Process(target=_overlap_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=240)
        assert p.exitcode == 0
    assert q.get(timeout=10)


@pytest.mark.parametrize("P", [1, 2, 3, 8])
def test_bench_shard_bytes_add_up(P):
    """bench.py's per-rank byte model (shard_kernel_bytes): SpMM bytes of the P row
    shards sum to the single-GPU SpMM bytes exactly; SDDMM bytes of the P edge shards
    sum to the single-GPU SDDMM bytes plus one A1 row (4K B) per row split between two
    edge shards -- the A1 term is not counted P times (round-1 overcount)."""
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    import bench
    import gen
    from paper_conf_ipps_fanwc23_b200 import dist as gdist
    g = gen.powerlaw_graph(3001, 60000, gamma=2.2, n_comm=5, seed=91)
    K = 64
    one = gdist.shard_spec(g.row_ptr, g.N, 0, 1)
    sp1, sd1, rows1 = bench.shard_kernel_bytes(g, one, K)
    assert rows1 == g.M and sp1 == bench.spmm_bytes(g.nnz, g.M, K)
    sp = sd = 0
    split = 0
    for r in range(P):
        s = gdist.shard_spec(g.row_ptr, g.N, r, P)
        a, b, _ = bench.shard_kernel_bytes(g, s, K)
        sp += a
        sd += b
        if r and s.f0 < g.nnz and s.f0 > 0 and g.row_ind[s.f0] == g.row_ind[s.f0 - 1]:
            split += 1
    assert sp == sp1
    assert sd == sd1 + split * 4 * K
