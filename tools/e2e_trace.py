"""Timeline of one gnn_run_host_multi call on C4 (GNN_HOST_TRACE=1: per-piece milestones
on the device clock), the e2e step time, the host enqueue time of the call, and the pure
copy floor for the same bytes (H2D and D2H pieces on two streams, no kernels)."""
import json
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_fanwc23_b200 as gs  # noqa: E402
from gen import configs  # noqa: E402


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "C4"
    Ks = [32, 64, 128, 256]
    g = configs.make_graph(name)
    runner = gs.HostRunner(g.M, g.N, g.row_ind, g.col_ind, g.val, max(Ks), Ks=Ks).pin()
    hX = [torch.from_numpy(configs.make_features(name, g.N, K)).pin_memory() for K in Ks]
    hO = [torch.empty((g.M, K)).pin_memory() for K in Ks]
    hE = [torch.empty(g.nnz).pin_memory() for _ in Ks]

    def step():
        runner.run_multi(hX, Ks, hO, hE, upload_graph=True)

    for _ in range(2):
        step()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    t0 = time.perf_counter()
    step()
    enq = time.perf_counter() - t0
    b.record()
    torch.cuda.synchronize()
    ms = a.elapsed_time(b)
    os.environ["GNN_HOST_TRACE"] = "1"
    step()
    torch.cuda.synchronize()
    del os.environ["GNN_HOST_TRACE"]

    # copy floor: the same H2D / D2H bytes in pieces on two streams
    h2d = 12 * g.nnz + sum(4 * g.N * K for K in Ks)
    d2h = sum(4 * g.M * K for K in Ks) + 4 * g.nnz * len(Ks)
    P = 28
    hs = torch.empty(h2d // 4 + 64).pin_memory()
    hd = torch.empty(d2h // 4 + 64).pin_memory()
    ds = torch.empty_like(hs, device="cuda")
    dd = torch.empty_like(hd, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

    def copies(up, down):
        a.record()
        s1.wait_event(a)
        s2.wait_event(a)
        n1, n2 = hs.numel(), hd.numel()
        for p in range(P):
            if up:
                with torch.cuda.stream(s1):
                    ds[n1 * p // P:n1 * (p + 1) // P].copy_(hs[n1 * p // P:n1 * (p + 1) // P], non_blocking=True)
            if down:
                with torch.cuda.stream(s2):
                    hd[n2 * p // P:n2 * (p + 1) // P].copy_(dd[n2 * p // P:n2 * (p + 1) // P], non_blocking=True)
        torch.cuda.current_stream().wait_stream(s1)
        torch.cuda.current_stream().wait_stream(s2)
        b.record()
        torch.cuda.synchronize()
        return a.elapsed_time(b)

    copies(1, 1)
    out = {"workload": name, "e2e_ms": round(ms, 3), "host_enqueue_ms": round(enq * 1e3, 3),
           "h2d_bytes": h2d, "d2h_bytes": d2h,
           "copy_floor_ms": {"h2d_only": round(copies(1, 0), 3), "d2h_only": round(copies(0, 1), 3),
                             "both": round(copies(1, 1), 3)}}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
