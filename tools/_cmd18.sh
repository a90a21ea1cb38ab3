mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -x > gpurun_out/pytest_gpu18.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu18.txt
timeout 1500 python tools/sweep.py --workload C4 --reorder --reps 3 build/libgnnsparse_ref.so build/libgnnsparse_x.so > gpurun_out/sweep18.txt 2>&1
timeout 1500 python tools/sweep.py --workload C4 --reorder --reps 3 --dtype bf16 build/libgnnsparse_x.so >> gpurun_out/sweep18.txt 2>&1
