#!/bin/bash
# A/B of the kernels before/after the tile refactor on one box + C5 chunk sweep + PCIe probe.
mkdir -p gpurun_out
timeout 300 python tools/pcie_probe.py > gpurun_out/pcie.json 2>&1
L="build/libgnnsparse_orig.so build/libgnnsparse_cur.so build/libgnnsparse_orig.so build/libgnnsparse_cur.so"
timeout 900 python tools/sweep.py --workload C4 --reorder --K 32,64,128,256 $L > gpurun_out/sweep_ab_c4.txt 2> gpurun_out/sweep_ab_c4.err
for C in 128 256 512; do
  timeout 600 python tools/sweep.py --workload C5 --reorder --K 64,128,256 --force-chunk $C build/libgnnsparse_cur.so >> gpurun_out/sweep_c5_chunk.txt 2>> gpurun_out/sweep_c5_chunk.err
  timeout 600 python tools/sweep.py --workload C5 --reorder --dtype bf16 --K 256 --force-chunk $C build/libgnnsparse_cur.so >> gpurun_out/sweep_c5_chunk.txt 2>> gpurun_out/sweep_c5_chunk.err
done
