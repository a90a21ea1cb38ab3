mkdir -p gpurun_out
timeout 1500 python tools/sweep.py --workload C4 build/libgnnsparse_f2.so build/libgnnsparse_j.so build/libgnnsparse_k.so build/libgnnsparse_l.so > gpurun_out/sweep4.txt 2>&1
timeout 600 python bench.py --steps 3 --warmup 3 > gpurun_out/bench4.json 2> gpurun_out/bench4.err
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"spmm_kernel|sddmm_kernel" -c 4 -f -o gpurun_out/prof4 python tools/profile_one.py --workload C4 --K 32,256 > gpurun_out/ncu4.log 2>&1
