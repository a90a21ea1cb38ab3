"""C3 (sampled subgraphs, K = 128): time the native one-call step (gnn_plan_spmm_sddmm)
per subgraph with the DTP chunk (force_chunk = 0) and with forced chunk sizes, plus the
SpMM and SDDMM kernels alone.  Prints one JSON line per setting.

    python tools/c3_chunk_sweep.py [--graphs 20] [--chunks 0,32,64,128,256]
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
    ap.add_argument("--chunks", default="0,16,32,64,128,256")
    ap.add_argument("--reps", type=int, default=50)
    ap.add_argument("--K", type=int, default=128)
    ap.add_argument("--alphas", default="0", help="DTP alpha values (0 = library default 2)")
    ap.add_argument("--wpb", type=int, default=0, help="warps per block (0 = library default)")
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    K = a.K
    subs = []
    for t in range(a.graphs):
        g = configs.make_c3(t)
        dg = gs.DeviceGraph.from_arrays(g.M, g.N, g.row_ind, g.col_ind, g.val, g.row_ptr,
                                        device=dev)
        X = torch.from_numpy(configs.make_features("C3", g.N, K)).to(dev)
        subs.append((g, dg, X, torch.empty((g.M, K), device=dev), torch.empty(g.nnz, device=dev)))
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    stream = torch.cuda.current_stream()
    settings = [(fc, 0) for fc in (int(c) for c in a.chunks.split(","))]
    settings += [(0, int(al)) for al in a.alphas.split(",") if int(al) > 0]
    for fc, al in settings:
        run = gs.StepRunner(dev)
        run.opts.force_chunk = fc
        run.opts.alpha = al
        run.opts.warps_per_block = a.wpb
        for s in subs:
            run(s[1], s[2], s[3], s[4])
        torch.cuda.synchronize()
        per, spm, sdd, chunks = [], [], [], []
        for r in range(a.reps):
            for i, (g, dg, X, O, E) in enumerate(subs):
                flush.fill_(float(r))
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                run(dg, X, O, E)
                e1.record(stream)
                per.append((e0, e1))
        torch.cuda.synchronize()
        ms = statistics.mean(x.elapsed_time(y) for x, y in per)
        # kernels alone (plan built once, outside the events)
        for (g, dg, X, O, E) in subs:
            p = gs.plan(dg, K, force_chunk=fc, alpha=al, warps_per_block=a.wpb)
            chunks.append(p.info()["chunk"])
            for fn, acc in ((lambda: gs.spmm(p, dg, X, out=O), spm),
                            (lambda: gs.sddmm(p, dg, X, X, out=E), sdd)):
                ts = []
                for r in range(5):
                    flush.fill_(float(r))
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(stream)
                    fn()
                    e1.record(stream)
                    ts.append((e0, e1))
                torch.cuda.synchronize()
                acc.append(statistics.median(x.elapsed_time(y) for x, y in ts))
        print(json.dumps({"force_chunk": fc, "alpha": al or 2, "wpb": a.wpb, "step_ms": round(ms, 4),
                          "spmm_ms_mean": round(statistics.mean(spm), 4),
                          "sddmm_ms_mean": round(statistics.mean(sdd), 4),
                          "chunks": sorted(set(chunks))}), flush=True)


if __name__ == "__main__":
    main()
