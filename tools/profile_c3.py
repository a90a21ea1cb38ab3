"""One-call C3 steps (gnn_plan_spmm_sddmm) on a few resident subgraphs, for ncu captures.

    python tools/profile_c3.py [--graphs 3] [--K 128]
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
    ap.add_argument("--graphs", type=int, default=3)
    ap.add_argument("--K", type=int, default=128)
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    run = gs.StepRunner(dev)
    for t in range(a.graphs):
        g = configs.make_c3(t)
        dg = gs.DeviceGraph.from_arrays(g.M, g.N, g.row_ind, g.col_ind, g.val, g.row_ptr,
                                        device=dev)
        X = torch.from_numpy(configs.make_features("C3", g.N, a.K)).to(dev)
        O, E = torch.empty((g.M, a.K), device=dev), torch.empty(g.nnz, device=dev)
        run(dg, X, O, E)
        torch.cuda.synchronize()
        print(t, g.M, g.nnz, flush=True)


if __name__ == "__main__":
    main()
