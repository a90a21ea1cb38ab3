mkdir -p gpurun_out
timeout 1500 python tools/sweep.py --workload C4 --reorder --reps 3 build/libgnnsparse_ref.so build/libgnnsparse_v4.so build/libgnnsparse_ref.so build/libgnnsparse_v4.so > gpurun_out/sweep16.txt 2>&1
GNN_LIB_PATH=$PWD/build/libgnnsparse_ref.so timeout 900 ncu --set full --clock-control none -k regex:"sddmm_kernel" -c 2 -f -o gpurun_out/prof16_ref python tools/profile_one.py --workload C4 --reorder --K 128,256 > gpurun_out/ncu16a.log 2>&1
GNN_LIB_PATH=$PWD/build/libgnnsparse_v4.so timeout 900 ncu --set full --clock-control none -k regex:"sddmm_kernel" -c 2 -f -o gpurun_out/prof16_v4 python tools/profile_one.py --workload C4 --reorder --K 128,256 > gpurun_out/ncu16b.log 2>&1
