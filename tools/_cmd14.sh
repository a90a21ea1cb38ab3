mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 > gpurun_out/pytest_gpu14.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu14.txt
timeout 2000 python tools/sweep.py --workload C4 --reorder --reps 3 build/libgnnsparse_cur.so > gpurun_out/sweep14.txt 2>&1
timeout 2000 python tools/sweep.py --workload C4 --reorder --reps 3 --dtype bf16 build/libgnnsparse_cur.so >> gpurun_out/sweep14.txt 2>&1
