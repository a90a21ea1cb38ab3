mkdir -p gpurun_out
timeout 2000 python tools/sweep.py --workload C4 --reorder --reps 3 build/libgnnsparse_s1.so build/libgnnsparse_s2.so build/libgnnsparse_s3.so build/libgnnsparse_s4.so build/libgnnsparse_s5.so build/libgnnsparse_s6.so build/libgnnsparse_s7.so > gpurun_out/sweep8.txt 2>&1
