mkdir -p gpurun_out
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench13.json 2> gpurun_out/bench13.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches13.csv python tools/profile_one.py --workload C4 --reorder --K 32,64,128,256 > gpurun_out/ncu13_launch.log 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"spmm_kernel|sddmm_kernel" -c 8 -f -o gpurun_out/prof13 python tools/profile_one.py --workload C4 --reorder --K 32,64,128,256 > gpurun_out/ncu13.log 2>&1
