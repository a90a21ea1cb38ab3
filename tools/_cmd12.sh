mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -x > gpurun_out/pytest_gpu12.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu12.txt
timeout 2000 python tools/sweep.py --workload C4 --reorder --reps 3 build/libgnnsparse_ref.so build/libgnnsparse_t0.so build/libgnnsparse_t1.so > gpurun_out/sweep12.txt 2>&1
