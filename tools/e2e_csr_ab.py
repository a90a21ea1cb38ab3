"""e2e A/B: gnn_run_host_multi over C4+GCR (K = 32..256, host buffers, bench.py's e2e call)
with the graph uploaded as RowInd vs as CSR offsets decoded on the device, alternated on
one box.  Prints one JSON line (ms per call, CUDA events, mean of --reps after warm-up).

    python tools/e2e_csr_ab.py [--reps 5] [--rounds 3]
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--rounds", type=int, default=3)
    a = ap.parse_args()
    g0 = configs.make_graph("C4")
    perm, _, _ = gs.reorder_gcr(g0.row_ptr, g0.col_ind)
    rp, ri, ci, v = gs.permute_graph(g0.row_ptr, g0.col_ind, g0.val, perm)
    g = gen.Graph(g0.M, g0.N, rp, ri, ci, v)
    Ks = [32, 64, 128, 256]
    Xs = []
    for K in Ks:
        X = configs.make_features("C4", g.N, K)
        Xp = np.empty_like(X)
        Xp[perm] = X
        Xs.append(torch.from_numpy(Xp).pin_memory())
    Os = [torch.empty((g.M, K)).pin_memory() for K in Ks]
    Es = [torch.empty(g.nnz).pin_memory() for _ in Ks]
    runners = {"row_ind": gs.HostRunner(g.M, g.N, g.row_ind, g.col_ind, g.val, 256, Ks=Ks).pin(),
               "csr": gs.HostRunner(g.M, g.N, g.row_ind, g.col_ind, g.val, 256, Ks=Ks,
                                    row_ptr=g.row_ptr).pin()}
    res = {k: [] for k in runners}
    for rnd in range(a.rounds):
        for name, r in runners.items():
            for _ in range(2):
                r.run_multi(Xs, Ks, Os, Es, upload_graph=True)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(a.reps):
                r.run_multi(Xs, Ks, Os, Es, upload_graph=True)
            e1.record()
            torch.cuda.synchronize()
            res[name].append(round(e0.elapsed_time(e1) / a.reps, 3))
    print(json.dumps({"workload": "C4+GCR", "Ks": Ks, **{f"{k}_ms": v for k, v in res.items()}}))


if __name__ == "__main__":
    main()
