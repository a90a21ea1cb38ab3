#!/bin/bash
# SDDMM lane-split variants (GNN_SDDMM_R2_FROM) at small K, fp32 and bf16, C4 GCR.
mkdir -p gpurun_out
L="build/libgnnsparse_base.so build/libgnnsparse_r2f2.so build/libgnnsparse_r2f4.so build/libgnnsparse_base.so"
timeout 900 python tools/sweep.py --workload C4 --reorder --K 16,32,64 $L > gpurun_out/sweep_sddmm_f32.txt 2> gpurun_out/sweep_sddmm_f32.err
timeout 900 python tools/sweep.py --workload C4 --reorder --dtype bf16 --K 32,64,128 $L > gpurun_out/sweep_sddmm_bf16.txt 2> gpurun_out/sweep_sddmm_bf16.err
