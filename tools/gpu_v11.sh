#!/bin/bash
# v11: GPU tests, benches (C4 headline, C5, C3), launch list + ncu full of the headline kernels.
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as e; e.smoke()" > gpurun_out/smoke11.txt 2>&1; echo "rc=$?" >> gpurun_out/smoke11.txt
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest11.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest11.txt
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench11_c4.json 2> gpurun_out/bench11_c4.err
timeout 900 python bench.py --workload C5 --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench11_c5.json 2> gpurun_out/bench11_c5.err
timeout 900 python bench.py --workload C3 --steps 40 --warmup 5 --no-cpu > gpurun_out/bench11_c3.json 2> gpurun_out/bench11_c3.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches11.csv python tools/profile_one.py --workload C4 --reorder --K 32,64,128,256 > gpurun_out/ncu11_launch.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"spmm_kernel|sddmm_kernel" -c 8 -f -o gpurun_out/prof11_c4gcr python tools/profile_one.py --workload C4 --reorder --K 32,64,128,256 > gpurun_out/ncu11_full.log 2>&1
timeout 1200 ncu --set full --clock-control none --cache-control none -k regex:"sddmm_kernel" -c 1 -f -o gpurun_out/prof11_c4gcr_warm_sddmm256 python tools/profile_one.py --workload C4 --reorder --K 256 --reps 2 > gpurun_out/ncu11_warm.log 2>&1
