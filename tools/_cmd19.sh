mkdir -p gpurun_out
timeout 2500 python tools/sweep.py --workload C4 --reorder --reps 3 build/libgnnsparse_x.so build/libgnnsparse_y1.so build/libgnnsparse_y2.so build/libgnnsparse_y3.so build/libgnnsparse_y4.so build/libgnnsparse_y5.so > gpurun_out/sweep19.txt 2>&1
timeout 2500 python tools/sweep.py --workload C4 --reorder --reps 3 --dtype bf16 build/libgnnsparse_x.so build/libgnnsparse_y1.so build/libgnnsparse_y2.so build/libgnnsparse_y3.so build/libgnnsparse_y4.so build/libgnnsparse_y5.so >> gpurun_out/sweep19.txt 2>&1
