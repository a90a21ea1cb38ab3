mkdir -p gpurun_out
timeout 2000 python tools/sweep.py --workload C4 --reorder --reps 3 build/libgnnsparse_ref.so build/libgnnsparse_q0.so build/libgnnsparse_q2.so build/libgnnsparse_ref.so > gpurun_out/sweep11.txt 2>&1
