mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -x > gpurun_out/pytest_gpu9.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu9.txt
timeout 2000 python tools/sweep.py --workload C4 --reorder --reps 3 build/libgnnsparse_p0.so build/libgnnsparse_p1.so build/libgnnsparse_p2.so build/libgnnsparse_p3.so > gpurun_out/sweep9.txt 2>&1
