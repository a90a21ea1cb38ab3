#!/bin/bash
# ncu full captures (with source) of the K=32 kernels, fp32 and bf16 features, GCR-reordered C4.
mkdir -p gpurun_out
for dt in f32 bf16; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"spmm_kernel|sddmm_kernel" -c 2 -f -o gpurun_out/prof_k32_$dt python tools/profile_one.py --workload C4 --reorder --K 32 --dtype $dt > gpurun_out/ncu_k32_$dt.log 2>&1
done
