"""Run plan + SpMM + SDDMM once per K on one workload (for ncu captures).

    python tools/profile_one.py --workload C4 --K 32,256 [--reps 1]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_fanwc23_b200 as gs  # noqa: E402
from gen import configs  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="C4")
    ap.add_argument("--K", default="32,256")
    ap.add_argument("--reps", type=int, default=1)
    ap.add_argument("--scale", type=float, default=1.0)
    ap.add_argument("--reorder", action="store_true")
    ap.add_argument("--dtype", default="f32", choices=["f32", "bf16"])
    a = ap.parse_args()
    g = configs.make_graph(a.workload, a.scale)
    perm = None
    if a.reorder:
        import gen
        perm, _, _ = gs.reorder_gcr(g.row_ptr, g.col_ind)
        rp, ri, ci, v = gs.permute_graph(g.row_ptr, g.col_ind, g.val, perm)
        g = gen.Graph(g.M, g.N, rp, ri, ci, v)
    dg = gs.DeviceGraph.from_arrays(g.M, g.N, g.row_ind, g.col_ind, g.val, g.row_ptr)
    for K in [int(k) for k in a.K.split(",")]:
        X = torch.from_numpy(configs.make_features(a.workload, g.N, K)).cuda()
        if perm is not None:
            X = gs.permute_rows(X, torch.from_numpy(perm))
        if a.dtype == "bf16":
            X = X.to(torch.bfloat16)
        O = torch.empty((g.M, K), device="cuda")
        E = torch.empty(g.nnz, device="cuda")
        for _ in range(a.reps):
            p = gs.plan(dg, K, feature_dtype=gs.GNN_BF16 if a.dtype == "bf16" else gs.GNN_F32)
            gs.spmm(p, dg, X, out=O)
            gs.sddmm(p, dg, X, X, out=E)
        torch.cuda.synchronize()
        print(K, p.info(), flush=True)


if __name__ == "__main__":
    main()
