"""Our SpMM / SDDMM against cuSPARSE (through torch.sparse: CSR SpMM = torch.sparse.mm,
CSR SDDMM = torch.sparse.sampled_addmm) on the same device graph and features -- the B200
analogue of the paper's Table III speedups (HP-SpMM vs cuSPARSE CSR ALG2: 1.90x / 2.53x
full-graph on V100 / A30; HP-SDDMM vs cuSPARSE CSR SDDMM: 10.90x / 11.17x).
Kernel time only (CUDA events), L2 flushed before each launch, the two alternated rep by
rep.  cuSPARSE's SDDMM writes (X X^T) at the pattern without the v_i scaling -- the same
gathers and flops minus one multiply per edge.

    python tools/vs_cusparse.py [--workload C4] [--K 32,64,128,256] [--reps 5] [--no-reorder]
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


def timed(fn, flush, reps):
    out = []
    for _ in range(reps):
        flush.fill_(1.0)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        out.append(a.elapsed_time(b))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="C4")
    ap.add_argument("--K", default="32,64,128,256")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--no-reorder", dest="reorder", action="store_false")
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    g = configs.make_graph(a.workload)
    perm = None
    if a.reorder:
        perm, _, _ = gs.reorder_gcr(g.row_ptr, g.col_ind)
        rp, ri, ci, v = gs.permute_graph(g.row_ptr, g.col_ind, g.val, perm)
        g = gen.Graph(g.M, g.N, rp, ri, ci, v)
    dg = gs.DeviceGraph.from_arrays(g.M, g.N, g.row_ind, g.col_ind, g.val, g.row_ptr, device=dev)
    S = torch.sparse_csr_tensor(torch.from_numpy(g.row_ptr).to(dev), torch.from_numpy(g.col_ind).to(dev),
                                torch.from_numpy(g.val).to(dev), size=(g.M, g.N))
    flush = torch.empty(256 * 1024 * 1024 // 4, device=dev)
    res = {"workload": a.workload, "reorder": a.reorder, "nnz": int(g.nnz),
           "cusparse": "torch %s, CSR int32 indices" % torch.__version__, "K": {}}
    for K in [int(k) for k in a.K.split(",")]:
        X = torch.from_numpy(configs.make_features(a.workload, g.N, K)).to(dev)
        if perm is not None:
            X = gs.permute_rows(X, torch.from_numpy(perm))
        XT = X.t()  # sampled_addmm(S, X, X^T): (X X^T) at S's pattern
        O = torch.empty((g.M, K), device=dev)
        E = torch.empty(g.nnz, device=dev)
        p = gs.plan(dg, K)
        ours_spmm = lambda: gs.spmm(p, dg, X, out=O)  # noqa: E731
        ours_sddmm = lambda: gs.sddmm(p, dg, X, X, out=E)  # noqa: E731
        cs_spmm = lambda: torch.sparse.mm(S, X)  # noqa: E731
        cs_sddmm = lambda: torch.sparse.sampled_addmm(S, X, XT, beta=0.0)  # noqa: E731
        for f in (ours_spmm, ours_sddmm, cs_spmm, cs_sddmm):
            f()
        torch.cuda.synchronize()
        # parity of the comparison itself: same SpMM result (fp32 rounding only)
        ref = cs_spmm()
        ours_spmm()
        torch.cuda.synchronize()
        rel = float((O - ref).abs().max() / ref.abs().max().clamp_min(1e-30))
        t = {k: [] for k in ("ours_spmm", "cusparse_spmm", "ours_sddmm", "cusparse_sddmm")}
        for _ in range(a.reps):
            t["ours_spmm"] += timed(ours_spmm, flush, 1)
            t["cusparse_spmm"] += timed(cs_spmm, flush, 1)
            t["ours_sddmm"] += timed(ours_sddmm, flush, 1)
            t["cusparse_sddmm"] += timed(cs_sddmm, flush, 1)
        med = {k: round(statistics.median(v), 4) for k, v in t.items()}
        res["K"][K] = {**{k + "_ms": v for k, v in med.items()},
                       "spmm_speedup": round(med["cusparse_spmm"] / med["ours_spmm"], 2),
                       "sddmm_speedup": round(med["cusparse_sddmm"] / med["ours_sddmm"], 2),
                       "spmm_max_rel_diff": rel}
        print(json.dumps({"K": K, **res["K"][K]}), flush=True)
        del X, O, E, p
        torch.cuda.empty_cache()
    print(json.dumps(res))


if __name__ == "__main__":
    main()
