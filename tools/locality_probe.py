"""SM-local traversal vs the kernels' chunk order, as pure gathers (tools/locality_probe.cu).

    make variants/liblocprobe.so && python tools/locality_probe.py [--workload C4] [--reps 5]

Prints one JSON line per (K, variant): ms (median over reps, the variants interleaved
round by round, L2 flushed before each) and the
gather rate n*(4K+4)/t -- the same byte count as bench.py's roofline probe.
"""
import argparse
import ctypes
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_fanwc23_b200 as gs  # noqa: E402
from gen import configs  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="C4")
    ap.add_argument("--Ks", default="32,64,128,256")
    ap.add_argument("--reps", type=int, default=9)
    ap.add_argument("--chunk", type=int, default=512)
    ap.add_argument("--front", action="store_true", help="also the batched persistent variants")
    ap.add_argument("--mlp", action="store_true", help="also loads-in-flight / occupancy variants")
    ap.add_argument("--smlocal", action="store_true", help="also the per-SM-range variants")
    a = ap.parse_args()
    lib = ctypes.CDLL(os.path.join(ROOT, "variants", "liblocprobe.so"))
    g0 = configs.make_graph(a.workload)
    perm, _, _ = gs.reorder_gcr(g0.row_ptr, g0.col_ind)
    rp, ri, ci, v = gs.permute_graph(g0.row_ptr, g0.col_ind, g0.val, perm)
    idx = torch.from_numpy(ci).cuda()
    n = idx.numel()
    sink = torch.zeros(1, device="cuda")
    nsm = torch.cuda.get_device_properties(0).multi_processor_count
    ctr = torch.zeros(2 * nsm, dtype=torch.int64, device="cuda")
    flush = torch.empty(64 * 1024 * 1024, device="cuda")
    st = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    for K in [int(k) for k in a.Ks.split(",")]:
        X = torch.from_numpy(configs.make_features(a.workload, g0.N, K)).cuda()
        variants = {"chunked": lambda: lib.lp_chunked(
            ctypes.c_void_p(X.data_ptr()), ctypes.c_int64(K), ctypes.c_void_p(idx.data_ptr()),
            ctypes.c_int64(n), K, a.chunk, ctypes.c_void_p(sink.data_ptr()), st)}
        for U, mb in ((2, 1), (4, 1), (8, 1), (2, 12), (4, 12), (2, 16), (4, 16), (8, 6),
                      (8, 9), (6, 9), (6, 12)) if a.mlp else ():
            variants[f"mlp_U{U}_minb{mb}"] = (lambda U=U, mb=mb: lib.lp_mlp(
                ctypes.c_void_p(X.data_ptr()), ctypes.c_int64(K), ctypes.c_void_p(idx.data_ptr()),
                ctypes.c_int64(n), K, a.chunk, U, mb, ctypes.c_void_p(sink.data_ptr()), st))
        for W in ((2, 4, 12, 18) if a.front else ()):
            for carve in (-1,):
                for ch in (a.chunk, a.chunk // 4):
                    variants[f"front_W{W}_chunk{ch}_carve{carve}"] = (
                        lambda W=W, cv=carve, ch=ch: lib.lp_front(
                            ctypes.c_void_p(X.data_ptr()), ctypes.c_int64(K),
                            ctypes.c_void_p(idx.data_ptr()), ctypes.c_int64(n), K, ch, W, cv,
                            ctypes.c_void_p(ctr.data_ptr()), ctypes.c_void_p(sink.data_ptr()), st))
        for KS in ((32, 64, 128, 256) if a.smlocal else ()):
            if KS > K:
                continue
            for bps in (8, 16):
                for sm_major in ((1, 0) if KS < K else (1,)):
                    for carve in (-1, 0):
                        name = f"smlocal_KS{KS}_b{bps}_{'slicemajor' if sm_major else 'chunkmajor'}_carve{carve}"
                        variants[name] = (lambda KS=KS, bps=bps, smj=sm_major, cv=carve: lib.lp_smlocal(
                            ctypes.c_void_p(X.data_ptr()), ctypes.c_int64(K),
                            ctypes.c_void_p(idx.data_ptr()), ctypes.c_int64(n), K, KS, a.chunk,
                            bps, smj, cv, ctypes.c_void_p(ctr.data_ptr()),
                            ctypes.c_void_p(sink.data_ptr()), st))
        for name, fn in variants.items():  # warm-up + launch check
            rc = fn()
            torch.cuda.synchronize()
            assert rc == 0, (name, rc)
        # variants interleaved round by round (clocks drift under the power cap): median
        ts = {name: [] for name in variants}
        for _ in range(a.reps):
            for name, fn in variants.items():
                flush.fill_(1.0)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                fn()
                e1.record()
                torch.cuda.synchronize()
                ts[name].append(e0.elapsed_time(e1))
        for name in variants:
            ms = statistics.median(ts[name])
            print(json.dumps({"workload": a.workload, "K": K, "variant": name, "ms": round(ms, 4),
                              "ms_min": round(min(ts[name]), 4),
                              "GBps": round(n * (4 * K + 4) / ms / 1e6, 1)}), flush=True)

if __name__ == "__main__":
    main()
