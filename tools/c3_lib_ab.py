"""C3 one-call step (gnn_plan_spmm_sddmm, K = 128) timed with several library builds,
alternated lib by lib in fresh subprocesses (GNN_LIB_PATH), same resident subgraphs, L2
flushed between steps, CUDA events around each step.  One JSON line per run.

    python tools/c3_lib_ab.py [--K 128] [--steps 2000] [--rounds 3] libA.so libB.so ...
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r'''
import json, os, statistics, sys
sys.path.insert(0, ROOT)
import torch
import paper_conf_ipps_fanwc23_b200 as gs
from gen import configs
dev = torch.device("cuda:0")
subs = []
for t in range(GRAPHS):
    g = configs.make_c3(t)
    dg = gs.DeviceGraph.from_arrays(g.M, g.N, g.row_ind, g.col_ind, g.val, g.row_ptr, device=dev)
    X = torch.from_numpy(configs.make_features("C3", g.N, K)).to(dev)
    subs.append((dg, X, torch.empty((g.M, K), device=dev), torch.empty(g.nnz, device=dev)))
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
stream = torch.cuda.current_stream()
run = gs.StepRunner(dev)
for s in subs:
    run(*s)
torch.cuda.synchronize()
ev = [[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in range(STEPS)]
for i in range(STEPS):
    flush.fill_(float(i))
    ev[i][0].record(stream)
    run(*subs[i % len(subs)])
    ev[i][1].record(stream)
torch.cuda.synchronize()
ts = [a.elapsed_time(b) for a, b in ev]
print("RESULT " + json.dumps({"lib": os.environ["GNN_LIB_PATH"], "K": K,
      "ms_mean": round(statistics.mean(ts), 5), "ms_median": round(statistics.median(ts), 5)}))
'''


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--K", type=int, default=128)
    ap.add_argument("--graphs", type=int, default=20)
    ap.add_argument("--steps", type=int, default=2000)
    ap.add_argument("--rounds", type=int, default=3)
    ap.add_argument("libs", nargs="+")
    a = ap.parse_args()
    code = f"K = {a.K}\n" + (CHILD.replace("ROOT", repr(ROOT)).replace("GRAPHS", str(a.graphs))
                               .replace("STEPS", str(a.steps)))
    for _ in range(a.rounds):
        for lib in a.libs:
            env = dict(os.environ, GNN_LIB_PATH=os.path.abspath(lib))
            r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True,
                               text=True, timeout=600)
            line = [l for l in r.stdout.splitlines() if l.startswith("RESULT ")]
            print(line[0][7:] if line else json.dumps({"lib": lib, "error": r.stderr[-1500:]}),
                  flush=True)


if __name__ == "__main__":
    main()
