"""Time SpMM / SDDMM of one or more library builds on one workload.

    python tools/sweep.py --workload C4 --K 32,64,128,256 build/libgnnsparse_a.so ...

Each library runs in its own subprocess (GNN_LIB_PATH), after a parity check on a
small graph against the oracle.  Prints one JSON line per library.
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r'''
import json, os, sys, time
sys.path.insert(0, ROOT)
import numpy as np, torch
import gen, oracle
import paper_conf_ipps_fanwc23_b200 as gs
from gen import configs
res = {"lib": os.environ["GNN_LIB_PATH"], "dtype": DTYPE, "force_chunk": FCHUNK, "wpb": WPB}
# parity on a small graph
g = gen.powerlaw_graph(4000, 200000, gamma=2.2, n_comm=5, seed=3)
dg = gs.DeviceGraph.from_arrays(g.M, g.N, g.row_ind, g.col_ind, g.val, g.row_ptr)
worst = 0.0
for K in (32, 64, 128, 256):
    X = gen.features(5, g.N, K)
    p = gs.plan(dg, K)
    O = gs.spmm(p, dg, torch.from_numpy(X).cuda()).cpu().numpy()
    E = gs.sddmm(p, dg, torch.from_numpy(X).cuda(), torch.from_numpy(X).cuda()).cpu().numpy()
    r, T = oracle.spmm(g.row_ind, g.col_ind, g.val, X, M=g.M)
    r2, T2 = oracle.sddmm(g.row_ind, g.col_ind, g.val, X, X)
    worst = max(worst, float((np.abs(O - r) / np.maximum(T, 1e-300)).max()),
                float((np.abs(E - r2) / np.maximum(T2, 1e-300)).max()))
res["parity_worst_err_over_T"] = worst
perm = None
cache = os.environ.get("GNN_SWEEP_CACHE")  # per-session scratch: the graph is deterministic
cfile = cache and os.path.join(cache, f"{WL}_{int(REORDER)}.npz")
if cfile and os.path.exists(cfile):
    z = np.load(cfile)
    g = gen.Graph(int(z["M"]), int(z["N"]), z["rp"], z["ri"], z["ci"], z["v"])
    perm = z["perm"] if REORDER else None
else:
    g = configs.make_graph(WL)
    if REORDER:
        perm, comm, q = gs.reorder_gcr(g.row_ptr, g.col_ind)
        rp, ri, ci, v = gs.permute_graph(g.row_ptr, g.col_ind, g.val, perm)
        g = gen.Graph(g.M, g.N, rp, ri, ci, v)
        res["modularity"] = q
    if cfile:
        os.makedirs(cache, exist_ok=True)
        np.savez(cfile, M=g.M, N=g.N, rp=g.row_ptr, ri=g.row_ind, ci=g.col_ind, v=g.val,
                 perm=perm if perm is not None else np.zeros(0, np.int32))
dg = gs.DeviceGraph.from_arrays(g.M, g.N, g.row_ind, g.col_ind, g.val, g.row_ptr)
flush = torch.empty(64 * 1024 * 1024, device="cuda")
for K, fvw in ([(k, 0) for k in KS] + [(k, 8) for k in KS if VW8 and k % 8 == 0 and k < 256]
                + [(k, ALTVW) for k in KS if ALTVW and k % ALTVW == 0]):
    X = torch.from_numpy(configs.make_features(WL, g.N, K)).cuda()
    if perm is not None:
        X = gs.permute_rows(X, torch.from_numpy(perm))
    if DTYPE == "bf16":
        X = X.to(torch.bfloat16)
    O = torch.empty((g.M, K), device="cuda"); E = torch.empty(g.nnz, device="cuda")
    p = gs.plan(dg, K, force_vw=fvw, feature_dtype=DTYPE, force_chunk=FCHUNK, warps_per_block=WPB)
    ts, td = [], []
    for it in range(REPS + 2):
        flush.fill_(it)
        a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        a.record(); gs.spmm(p, dg, X, out=O); b.record(); gs.sddmm(p, dg, X, X, out=E); c.record()
        torch.cuda.synchronize()
        if it >= 2:
            ts.append(a.elapsed_time(b)); td.append(b.elapsed_time(c))
    res[f"K{K}" + (f"_vw{fvw}" if fvw else "")] = {"spmm_ms": round(min(ts), 4), "sddmm_ms": round(min(td), 4),
                    "spmm_med": round(sorted(ts)[len(ts)//2], 4), "info": {k: p.info()[k] for k in ("chunk", "active_blocks_per_sm", "warps_per_block")}}
print("RESULT " + json.dumps(res), flush=True)
'''


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="C4")
    ap.add_argument("--K", default="32,64,128,256")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--vw8", action="store_true")
    ap.add_argument("--alt-vw", type=int, default=0,
                    help="also time every K with force_vw = this (elements per feature load)")
    ap.add_argument("--reorder", action="store_true")
    ap.add_argument("--dtype", default="f32", choices=["f32", "bf16"])
    ap.add_argument("--force-chunk", type=int, default=0)
    ap.add_argument("--wpb", type=int, default=0, help="plan warps_per_block (0 = default 8)")
    ap.add_argument("libs", nargs="+")
    a = ap.parse_args()
    code = CHILD.replace("ROOT", repr(ROOT)).replace("WL", repr(a.workload)).replace(
        "KS", repr([int(k) for k in a.K.split(",")])).replace("REPS", str(a.reps)).replace("VW8", str(a.vw8)).replace("REORDER", str(a.reorder)).replace("DTYPE", repr(a.dtype)).replace("FCHUNK", str(a.force_chunk)).replace("ALTVW", str(a.alt_vw)).replace("WPB", str(a.wpb))
    for lib in a.libs:
        env = dict(os.environ, GNN_LIB_PATH=os.path.abspath(lib))
        r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True,
                           timeout=900)
        line = [l for l in r.stdout.splitlines() if l.startswith("RESULT ")]
        if line:
            print(line[0][7:], flush=True)
        else:
            print(json.dumps({"lib": lib, "error": (r.stderr or r.stdout)[-2000:]}), flush=True)


if __name__ == "__main__":
    main()
