#!/bin/bash
# v13 (session 3): HEAD re-verified -- smoke, GPU tests, benches (C4 headline, C5, C3),
# launch list + ncu full of the headline kernels (exported to CSV on the box: the
# .ncu-rep files are too large to bring back).
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/nvsmi13.txt 2>&1; nproc >> gpurun_out/nvsmi13.txt
timeout 300 python -c "import __graft_entry__ as e; e.smoke()" > gpurun_out/smoke13.txt 2>&1; echo "rc=$?" >> gpurun_out/smoke13.txt
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest13.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest13.txt
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench13_c4.json 2> gpurun_out/bench13_c4.err
timeout 900 python bench.py --workload C5 --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench13_c5.json 2> gpurun_out/bench13_c5.err
timeout 900 python bench.py --workload C3 --steps 40 --warmup 5 --no-cpu > gpurun_out/bench13_c3.json 2> gpurun_out/bench13_c3.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches13.csv python tools/profile_one.py --workload C4 --reorder --K 32,64,128,256 > gpurun_out/ncu13_launch.log 2>&1
ncu_full() {  # name, ncu args..., -- profile_one args
  local n=$1; shift
  timeout 1200 ncu --set full --clock-control none "$@" > gpurun_out/$n.log 2>&1
  ncu -i /tmp/$n.ncu-rep --page raw --csv > gpurun_out/$n.csv 2>> gpurun_out/$n.log
  rm -f /tmp/$n.ncu-rep
}
ncu_full prof13_c4gcr -k regex:"spmm_kernel|sddmm_kernel" -c 8 -f -o /tmp/prof13_c4gcr python tools/profile_one.py --workload C4 --reorder --K 32,64,128,256
ncu_full prof13_c4gcr_warm_sddmm256 --cache-control none -k regex:"sddmm_kernel" -c 1 -f -o /tmp/prof13_c4gcr_warm_sddmm256 python tools/profile_one.py --workload C4 --reorder --K 256 --reps 2
ncu_full prof13_c5gcr -k regex:"spmm_kernel|sddmm_kernel" -c 2 -f -o /tmp/prof13_c5gcr python tools/profile_one.py --workload C5 --reorder --K 256
du -sh gpurun_out
