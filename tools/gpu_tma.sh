#!/bin/bash
# TMA sparse-tile session: GPU tests on the default build, then a variant sweep.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider -x > gpurun_out/pytest_tma.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_tma.txt
L="build/libgnnsparse_async.so build/libgnnsparse_tm1.so build/libgnnsparse_tm2.so build/libgnnsparse_tm4.so"
timeout 900 python tools/sweep.py --workload C4 --reorder --K 32,64,128,256 $L > gpurun_out/sweep_tma_c4.txt 2> gpurun_out/sweep_tma_c4.err
timeout 900 python tools/sweep.py --workload C4 --reorder --dtype bf16 --K 32,64,128,256 $L > gpurun_out/sweep_tma_c4bf16.txt 2> gpurun_out/sweep_tma_c4bf16.err
timeout 900 python tools/sweep.py --workload C5 --reorder --K 256 $L > gpurun_out/sweep_tma_c5.txt 2> gpurun_out/sweep_tma_c5.err
