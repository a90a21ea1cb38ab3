mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q --timeout 600 > gpurun_out/pytest_gpu6.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu6.txt
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench6.json 2> gpurun_out/bench6.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches6.csv python tools/profile_one.py --workload C4 --reorder --K 32,64,128,256 > gpurun_out/ncu6_launch.log 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"spmm_kernel|sddmm_kernel" -c 8 -f -o gpurun_out/prof6 python tools/profile_one.py --workload C4 --reorder --K 32,64,128,256 > gpurun_out/ncu6.log 2>&1
