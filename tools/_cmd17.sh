mkdir -p gpurun_out
timeout 1500 python tools/sweep.py --workload C4 --reorder --reps 3 build/libgnnsparse_ref.so build/libgnnsparse_w.so > gpurun_out/sweep17.txt 2>&1
timeout 1500 python tools/sweep.py --workload C4 --reorder --reps 3 --dtype bf16 build/libgnnsparse_w.so >> gpurun_out/sweep17.txt 2>&1
