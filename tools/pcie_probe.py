"""PCIe copy ceilings on the box: pinned H2D alone, D2H alone, and both directions at
once on two streams (what gnn_run_host_multi overlaps).  One JSON line."""
import json

import torch


def main():
    n = 512 << 20  # bytes per buffer
    h_src = torch.empty(n, dtype=torch.uint8).pin_memory()
    h_dst = torch.empty(n, dtype=torch.uint8).pin_memory()
    d_a = torch.empty(n, dtype=torch.uint8, device="cuda")
    d_b = torch.empty(n, dtype=torch.uint8, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

    def run(h2d, d2h, reps=5):
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(reps):
            if h2d:
                s1.wait_event(a)
                with torch.cuda.stream(s1):
                    d_a.copy_(h_src, non_blocking=True)
            if d2h:
                s2.wait_event(a)
                with torch.cuda.stream(s2):
                    h_dst.copy_(d_b, non_blocking=True)
        torch.cuda.current_stream().wait_stream(s1)
        torch.cuda.current_stream().wait_stream(s2)
        b.record()
        torch.cuda.synchronize()
        return reps * n * (h2d + d2h) / (a.elapsed_time(b) * 1e-3) / 1e9

    run(1, 1, 1)
    out = {"h2d_GBps": round(run(1, 0), 1), "d2h_GBps": round(run(0, 1), 1),
           "duplex_total_GBps": round(run(1, 1), 1), "bytes_per_copy": n}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
