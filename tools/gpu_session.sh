#!/bin/bash
# One GPU session: smoke, gpu tests, bench, ncu launch list + full captures.
# usage: tools/gpu_session.sh [tests|bench|ncu|all]...
mkdir -p gpurun_out
what="${@:-all}"
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/nvsmi.txt 2>&1
nproc >> gpurun_out/nvsmi.txt
for w in $what; do
case $w in
  smoke|all)
    timeout 300 python -c "import __graft_entry__ as e; e.smoke()" > gpurun_out/smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.txt ;;&
  tests|all)
    timeout 1500 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt ;;&
  bench|all)
    timeout 900 python bench.py --steps 3 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err ;;&
  ncu|all)
    timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python tools/profile_one.py --workload C4 --K 32,64,128,256 > gpurun_out/ncu_launch.log 2>&1
    timeout 1200 ncu --set full --clock-control none --import-source on -k regex:spmm_kernel -c 2 -f -o gpurun_out/prof_spmm python tools/profile_one.py --workload C4 --K 32,256 > gpurun_out/ncu_spmm.log 2>&1
    timeout 1200 ncu --set full --clock-control none --import-source on -k regex:sddmm_kernel -c 2 -f -o gpurun_out/prof_sddmm python tools/profile_one.py --workload C4 --K 32,256 > gpurun_out/ncu_sddmm.log 2>&1 ;;
esac
done
ls -la gpurun_out
