#!/bin/bash
mkdir -p gpurun_out
L="build/libgnnsparse_base.so build/libgnnsparse_vst.so build/libgnnsparse_base.so build/libgnnsparse_vst.so"
timeout 900 python tools/sweep.py --workload C4 --reorder --K 16,32,64 $L > gpurun_out/sweep_vst_f32.txt 2> gpurun_out/sweep_vst_f32.err
timeout 900 python tools/sweep.py --workload C4 --reorder --dtype bf16 --K 32,64,128 $L > gpurun_out/sweep_vst_bf16.txt 2> gpurun_out/sweep_vst_bf16.err
timeout 900 python tools/sweep.py --workload C5 --reorder --K 32,64 build/libgnnsparse_base.so build/libgnnsparse_vst.so > gpurun_out/sweep_vst_c5.txt 2> gpurun_out/sweep_vst_c5.err
