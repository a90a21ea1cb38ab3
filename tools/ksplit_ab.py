"""C4+GCR K=256 (X = 239 MB > 126 MB L2): one SpMM launch over all 256 columns vs two
launches over column halves (each half's X, 119 MB, nearly L2-resident: less DRAM
traffic, less power), each run sustained for --seconds so the GPU settles into its power
/ clock regime; CUDA-event time per SpMM pass and nvidia-smi clocks/power while running.

    python tools/ksplit_ab.py [--seconds 6] [--rounds 2]
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_fanwc23_b200 as gs  # noqa: E402
from gen import configs  # noqa: E402


def sample_clocks(seconds):
    p = subprocess.Popen(["nvidia-smi", "-i", "0", "--query-gpu=clocks.sm,power.draw",
                          "--format=csv,noheader,nounits", "-lms", "200"],
                         stdout=subprocess.PIPE, text=True)
    return p


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--seconds", type=float, default=6.0)
    ap.add_argument("--rounds", type=int, default=2)
    a = ap.parse_args()
    g0 = configs.make_graph("C4")
    perm, _, _ = gs.reorder_gcr(g0.row_ptr, g0.col_ind)
    rp, ri, ci, v = gs.permute_graph(g0.row_ptr, g0.col_ind, g0.val, perm)
    g = gen.Graph(g0.M, g0.N, rp, ri, ci, v)
    dg = gs.DeviceGraph.from_arrays(g.M, g.N, g.row_ind, g.col_ind, g.val, g.row_ptr)
    X = torch.from_numpy(configs.make_features("C4", g.N, 256)).cuda()
    O = torch.empty((g.M, 256), device="cuda")
    p256 = gs.plan(dg, 256)
    p128 = gs.plan(dg, 128, force_chunk=p256.info()["chunk"])
    halves = [(X[:, :128], O[:, :128]), (X[:, 128:], O[:, 128:])]
    variants = {
        "one_launch_K256": lambda: gs.spmm(p256, dg, X, out=O),
        "two_launches_K128_halves": lambda: [gs.spmm(p128, dg, x, out=o) for x, o in halves],
    }
    res = {k: [] for k in variants}
    for rnd in range(a.rounds):
        for name, fn in variants.items():
            for _ in range(3):
                fn()
            torch.cuda.synchronize()
            mon = sample_clocks(a.seconds)
            ts = []
            t_end = time.time() + a.seconds
            while time.time() < t_end:
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                fn()
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            mon.terminate()
            out = mon.communicate()[0].strip().splitlines()
            clk = [float(l.split(",")[0]) for l in out if l.strip()]
            pw = [float(l.split(",")[1]) for l in out if l.strip()]
            res[name].append({"ms_median": round(statistics.median(ts), 4), "n": len(ts),
                              "sm_mhz_median": statistics.median(clk) if clk else None,
                              "power_w_median": statistics.median(pw) if pw else None})
    print(json.dumps(res))


if __name__ == "__main__":
    main()
