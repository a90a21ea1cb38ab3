"""Measured peaks on this B200 (run under gpurun): HBM copy and random-row gather
from L1-, L2- and HBM-resident feature matrices, K = 32..256.  Writes one JSON line.

    python tools/microbench.py > profiles/<tag>_microbench.json
"""
import ctypes
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
lib = ctypes.CDLL(os.path.join(ROOT, "variants", "libgnnmicro.so"))
vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
lib.mb_gather.argtypes = [vp, i64, vp, i64, i32, vp, vp, i32]
lib.mb_copy.argtypes = [vp, vp, i64, vp, i32]
lib.mb_shfl.argtypes = [i32, i32, vp, vp]
lib.mb_fma.argtypes = [i32, i32, i32, vp, vp]


def timed(fn, reps=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    best = 1e9
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b))
    return best


def main():
    dev = torch.device("cuda")
    nsm = torch.cuda.get_device_properties(0).multi_processor_count
    st = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    res = {"gpu": torch.cuda.get_device_name(0), "sms": nsm,
           "l2_bytes": torch.cuda.get_device_properties(0).L2_cache_size}
    nbytes = 4 << 30
    a = torch.empty(nbytes // 4, device=dev)
    b = torch.empty(nbytes // 4, device=dev)
    ms = timed(lambda: lib.mb_copy(vp(a.data_ptr()), vp(b.data_ptr()), nbytes, st, nsm * 8))
    res["hbm_copy_GBps"] = round(2 * nbytes / ms / 1e6, 1)
    del a, b
    n = 64 * 1024 * 1024  # gathers per launch
    out = torch.zeros(1, device=dev)
    res["gather"] = {}
    for K in (32, 64, 128, 256):
        for tier, rows in (("L1", 256), ("L2", (32 << 20) // (4 * K)), ("HBM", (4 << 30) // (4 * K))):
            X = torch.randn(rows, K, device=dev)
            idx = torch.randint(0, rows, (n,), device=dev, dtype=torch.int32)
            for blocks_per_sm in (8, 16):
                ms = timed(lambda: lib.mb_gather(vp(X.data_ptr()), K, vp(idx.data_ptr()), n, K,
                                                 vp(out.data_ptr()), st, nsm * blocks_per_sm), reps=5)
                gbps = n * 4 * K / ms / 1e6
                key = f"K{K}_{tier}"
                res["gather"][key] = max(res["gather"].get(key, 0), round(gbps, 1))
            del X, idx
    # warp-shuffle issue rate: warp-wide SHFL instructions per SM per clock
    blocks, iters = nsm * 8, 4096
    ms = timed(lambda: lib.mb_shfl(blocks, iters, vp(out.data_ptr()), st))
    warps = blocks * 8
    res["shfl_warp_instr_per_s"] = round(warps * iters * 8 / (ms * 1e-3), 1)
    res["shfl_per_sm_per_clk_at_1965MHz"] = round(warps * iters * 8 / (ms * 1e-3) / nsm / 1.965e9, 3)
    # fp32 FMA throughput: scalar FFMA vs packed FFMA2 (SURVEY §8(d) peak #4)
    res["fma"] = {}
    for packed, tag in ((0, "FFMA"), (1, "FFMA2")):
        ms = timed(lambda: lib.mb_fma(packed, blocks, iters, vp(out.data_ptr()), st))
        flops = blocks * 256 * iters * 32 * 2
        res["fma"][tag] = {"TFLOPs": round(flops / (ms * 1e-3) / 1e12, 2),
                           "fma_per_sm_per_clk_at_1965MHz":
                               round(flops / 2 / (ms * 1e-3) / nsm / 1.965e9, 1)}
    print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
