"""SpMM lane-mapping experiment (round-1 verdict item 8): interleaved lane groups with a
warp-shuffle reduction at row ends (tools/spmm_interleaved.cu) vs the same memory code
with each group walking its own chunk, vs the product kernel (gs.spmm).  Both experiment
kernels zero O with a memset first (its time is reported and subtracted).  Outputs are
checked against the product's.  One JSON line per (workload, K).

    python tools/interleaved_ab.py [--c3-graphs 20]
"""
import argparse
import ctypes
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_fanwc23_b200 as gs  # noqa: E402
from gen import configs  # noqa: E402

EXP = ctypes.CDLL(os.path.join(ROOT, "variants", "libgnnexp.so"))
vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
for f in (EXP.exp_spmm_interleaved, EXP.exp_spmm_ownchunk):
    f.argtypes = [vp, vp, vp, i64, i64, i32, i32, vp, i64, vp, i64, i32, vp]
    f.restype = ctypes.c_int


def run_exp(fn, dg, K, C, X, O, zero=1):
    st = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    rc = fn(dg.row_ind.data_ptr(), dg.col_ind.data_ptr(),
            None if dg.val is None else dg.val.data_ptr(), dg.nnz, dg.M, K, C, X.data_ptr(),
            X.stride(0), O.data_ptr(), O.stride(0), zero, st)
    assert rc == 0, rc


def timed(fns, reps, flush):
    """mean ms of running every fn in fns (one step) over reps steps, L2 flushed between."""
    ts = []
    for it in range(reps + 2):
        flush.fill_(float(it))
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for f in fns:
            f()
        b.record()
        torch.cuda.synchronize()
        if it >= 2:
            ts.append(a.elapsed_time(b))
    return statistics.mean(ts)


def measure(name, graphs, K, reps, flush):
    ent = []
    for g in graphs:
        dg = gs.DeviceGraph.from_arrays(g.M, g.N, g.row_ind, g.col_ind, g.val, g.row_ptr)
        X = torch.from_numpy(configs.make_features("C3" if name == "C3" else name, g.N, K)).cuda()
        p = gs.plan(dg, K)
        C = p.info()["chunk"]
        Op, Oi, Oo = (torch.empty((g.M, K), device="cuda") for _ in range(3))
        ent.append((dg, X, p, C, Op, Oi, Oo))
    # correctness against the product kernel
    worst = 0.0
    for dg, X, p, C, Op, Oi, Oo in ent:
        gs.spmm(p, dg, X, out=Op)
        run_exp(EXP.exp_spmm_interleaved, dg, K, C, X, Oi)
        run_exp(EXP.exp_spmm_ownchunk, dg, K, C, X, Oo)
        torch.cuda.synchronize()
        scale = Op.abs().amax(dim=1, keepdim=True).clamp_min(1e-30)
        for Ox in (Oi, Oo):
            d = ((Ox - Op).abs() / scale).max().item()
            worst = max(worst, d if np.isfinite(d) else float("inf"))  # NaN fails loudly
        worst = max(worst, 0.0 if bool(torch.isfinite(Op).all()) else float("inf"))
    nonfinite = [int((~torch.isfinite(t)).sum()) for t in (ent[0][4], ent[0][5], ent[0][6])]
    e0 = ent[0]
    dbg = {"sum_abs_product": float(e0[4].abs().sum()),
           "sum_abs_diff_interleaved": float((e0[5] - e0[4]).abs().sum()),
           "sum_abs_diff_own": float((e0[6] - e0[4]).abs().sum()),
           "frac_elems_differing_interleaved": float((e0[5] != e0[4]).float().mean()),
           "sample": [float(e0[4][0, 0]), float(e0[5][0, 0]), float(e0[6][0, 0])]}
    res = {"workload": name, "K": K, "graphs": len(ent), "chunk": sorted({e[3] for e in ent}),
           "max_rel_diff_vs_product": worst,
           "nonfinite_product_interleaved_ownchunk": nonfinite, "debug": dbg}
    res["product_ms"] = timed([lambda e=e: gs.spmm(e[2], e[0], e[1], out=e[4]) for e in ent],
                              reps, flush) / len(ent)
    res["memset_ms"] = timed([lambda e=e: e[5].zero_() for e in ent], reps, flush) / len(ent)
    for tag, fn in (("interleaved", EXP.exp_spmm_interleaved), ("own_chunk", EXP.exp_spmm_ownchunk)):
        ms = timed([lambda e=e: run_exp(fn, e[0], K, e[3], e[1], e[5]) for e in ent], reps,
                   flush) / len(ent)
        res[f"{tag}_ms_incl_memset"] = ms
        res[f"{tag}_ms"] = ms - res["memset_ms"]
    out = {k: (round(v, 4) if isinstance(v, float) else v) for k, v in res.items()}
    out["max_rel_diff_vs_product"] = float(f"{worst:.3e}")  # rounding-level (~1e-7)
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--c3-graphs", type=int, default=20)
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--quick", action="store_true", help="C3 only")
    a = ap.parse_args()
    flush = torch.empty(64 * 1024 * 1024, device="cuda")
    c3 = [configs.make_c3(t) for t in range(a.c3_graphs)]
    for K in (32, 64, 128):
        print(json.dumps(measure("C3", c3, K, a.reps, flush)), flush=True)
    if a.quick:
        return
    del c3
    for name, Ks in (("C4", (32, 64, 128)), ("C5", (64, 128, 256))):
        g0 = configs.make_graph(name)
        perm, _, _ = gs.reorder_gcr(g0.row_ptr, g0.col_ind)
        rp, ri, ci, v = gs.permute_graph(g0.row_ptr, g0.col_ind, g0.val, perm)
        g = gen.Graph(g0.M, g0.N, rp, ri, ci, v)
        del g0
        for K in Ks:
            print(json.dumps(measure(name, [g], K, max(3, a.reps // 4), flush)), flush=True)
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
