mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 > gpurun_out/pytest_gpu20.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu20.txt
timeout 300 python -c "import __graft_entry__ as e; e.smoke()" > gpurun_out/smoke20.txt 2>&1; echo "rc=$?" >> gpurun_out/smoke20.txt
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench20.json 2> gpurun_out/bench20.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches20.csv python tools/profile_one.py --workload C4 --reorder --K 32,64,128,256 > gpurun_out/ncu20_launch.log 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"spmm_kernel|sddmm_kernel" -c 8 -f -o gpurun_out/prof20 python tools/profile_one.py --workload C4 --reorder --K 32,64,128,256 > gpurun_out/ncu20.log 2>&1
