mkdir -p gpurun_out
timeout 2000 python tools/sweep.py --workload C4 --reorder --reps 3 build/libgnnsparse_q0.so build/libgnnsparse_q1.so build/libgnnsparse_q2.so > gpurun_out/sweep10.txt 2>&1
