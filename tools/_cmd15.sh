mkdir -p gpurun_out
timeout 2500 python tools/sweep.py --workload C4 --reorder --reps 3 build/libgnnsparse_ref.so build/libgnnsparse_v4.so build/libgnnsparse_v2.so build/libgnnsparse_v1.so > gpurun_out/sweep15.txt 2>&1
timeout 2000 python tools/sweep.py --workload C4 --reorder --reps 3 --dtype bf16 build/libgnnsparse_v4.so build/libgnnsparse_v2.so build/libgnnsparse_v1.so >> gpurun_out/sweep15.txt 2>&1
