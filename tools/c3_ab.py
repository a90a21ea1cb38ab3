"""C3 (sampled subgraphs, K = 128) one-call step A/B/C: gnn_plan_spmm_sddmm as one fused
SpMM+SDDMM launch (default), as two kernels on two streams with the boundary table
recomputed in-kernel (GNN_STEP_FUSED=0), and with the plan kernel (GNN_STEP_PLAN_KERNEL=1),
alternated on the same resident subgraphs, L2 flushed between steps, CUDA events around
each step.  Prints one JSON line.

    python tools/c3_ab.py [--graphs 20] [--steps 2000] [--rounds 3]
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_fanwc23_b200 as gs  # noqa: E402
from gen import configs  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--graphs", type=int, default=20)
    ap.add_argument("--steps", type=int, default=2000)
    ap.add_argument("--rounds", type=int, default=3)
    ap.add_argument("--K", type=int, default=128)
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    K = a.K
    subs = []
    for t in range(a.graphs):
        g = configs.make_c3(t)
        dg = gs.DeviceGraph.from_arrays(g.M, g.N, g.row_ind, g.col_ind, g.val, g.row_ptr,
                                        device=dev)
        X = torch.from_numpy(configs.make_features("C3", g.N, K)).to(dev)
        subs.append((dg, X, torch.empty((g.M, K), device=dev), torch.empty(g.nnz, device=dev)))
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    stream = torch.cuda.current_stream()
    run = gs.StepRunner(dev)
    # (GNN_STEP_FUSED, GNN_STEP_PLAN_KERNEL)
    modes = {"fused": ("1", "0"), "two_kernels": ("0", "0"), "plan_kernel": ("0", "1")}
    res = {m: [] for m in modes}
    for rnd in range(a.rounds):
        for mode, (fz, pk) in modes.items():
            os.environ["GNN_STEP_FUSED"] = fz
            os.environ["GNN_STEP_PLAN_KERNEL"] = pk
            for s in subs:
                run(*s)
            torch.cuda.synchronize()
            ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                  for _ in range(a.steps)]
            for i in range(a.steps):
                flush.fill_(float(i))
                ev[i][0].record(stream)
                run(*subs[i % len(subs)])
                ev[i][1].record(stream)
            torch.cuda.synchronize()
            res[mode].append(statistics.mean(x.elapsed_time(y) for x, y in ev))
    os.environ.pop("GNN_STEP_PLAN_KERNEL", None)
    os.environ.pop("GNN_STEP_FUSED", None)
    print(json.dumps({"K": K, "graphs": a.graphs, "steps": a.steps,
                      **{f"{m}_ms": [round(x, 4) for x in v] for m, v in res.items()}}))


if __name__ == "__main__":
    main()
