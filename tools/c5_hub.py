"""C5 (products-shaped, X = 2.5 GB >> L2) DRAM over-fetch experiments, K = 256:
GCR order with a hub block of H rows first (reorder_gcr(hub_rows=H)) x gathers of that
block with an L2 evict_last policy (plan option hub_rows of the library at commit 084431e;
the hint measured slower and was removed, profiles/r02_s3_c5_hub.txt -- with later
libraries only hint = 0 runs), and SpMM split into two K = 128 column halves (half the
bytes per row in flight).  SpMM / SDDMM timed with CUDA events,
L2 flushed between runs, median of --reps.  One JSON line per setting.

    python tools/c5_hub.py [--hubs 0,32768,65536] [--reps 5] [--profile H:hint]
"""
import argparse
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


def timed(fn, reps, flush):
    ts = []
    for it in range(reps + 1):
        flush.fill_(float(it))
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        if it:
            ts.append(a.elapsed_time(b))
    return round(statistics.median(ts), 4)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="C5")
    ap.add_argument("--K", type=int, default=256)
    ap.add_argument("--hubs", default="0,32768,65536")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--dtype", default="f32")
    ap.add_argument("--profile", default="", help="H:hint -- run once for ncu, no timing")
    a = ap.parse_args()
    K = a.K
    g0 = configs.make_graph(a.workload)
    X0 = configs.make_features(a.workload, g0.N, K)
    flush = torch.empty(64 * 1024 * 1024, device="cuda")
    hubs = [int(h) for h in a.hubs.split(",")]
    if a.profile:
        h, hint = (int(x) for x in a.profile.split(":"))
        hubs = [h]
    for H in hubs:
        perm, _, _ = gs.reorder_gcr(g0.row_ptr, g0.col_ind, hub_rows=H)
        rp, ri, ci, v = gs.permute_graph(g0.row_ptr, g0.col_ind, g0.val, perm)
        g = gen.Graph(g0.M, g0.N, rp, ri, ci, v)
        dg = gs.DeviceGraph.from_arrays(g.M, g.N, g.row_ind, g.col_ind, g.val, g.row_ptr)
        Xp = np.empty_like(X0)
        Xp[perm] = X0
        X = torch.from_numpy(Xp).cuda()
        if a.dtype == "bf16":
            X = X.to(torch.bfloat16)
        O = torch.empty((g.M, K), device="cuda")
        E = torch.empty(g.nnz, device="cuda")
        has_hint = "hub_rows" in dict(gs.PlanOpts._fields_)
        for hint in ([0, 1] if H and has_hint else [0]):
            if a.profile and hint != int(a.profile.split(":")[1]):
                continue
            kw = {"hub_rows": H} if hint else {}
            p = gs.plan(dg, K, feature_dtype=a.dtype, **kw)
            if a.profile:
                gs.spmm(p, dg, X, out=O)
                gs.sddmm(p, dg, X, X, out=E)
                torch.cuda.synchronize()
                print(json.dumps({"profiled": H, "hint": hint}), flush=True)
                continue
            res = {"workload": a.workload, "K": K, "dtype": a.dtype, "hub_rows": H,
                   "hint": hint, "chunk": p.info()["chunk"]}
            res["spmm_ms"] = timed(lambda: gs.spmm(p, dg, X, out=O), a.reps, flush)
            res["sddmm_ms"] = timed(lambda: gs.sddmm(p, dg, X, X, out=E), a.reps, flush)
            if K % 2 == 0 and a.dtype == "f32":
                # K-split: two launches over column halves (pitched views, same graph)
                ph = gs.plan(dg, K // 2, **kw)
                Xa, Xb = X[:, :K // 2], X[:, K // 2:]
                Oa, Ob = O[:, :K // 2], O[:, K // 2:]

                def ksplit():
                    gs.spmm(ph, dg, Xa, out=Oa)
                    gs.spmm(ph, dg, Xb, out=Ob)
                res["spmm_ksplit_ms"] = timed(ksplit, a.reps, flush)
            print(json.dumps(res), flush=True)
        del X, O, E, dg
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
