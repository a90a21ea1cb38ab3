mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q --timeout 600 -x > gpurun_out/pytest_gpu2.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu2.txt
timeout 1500 python tools/sweep.py --workload C4 build/libgnnsparse_a.so build/libgnnsparse_b.so build/libgnnsparse_c.so build/libgnnsparse_d.so build/libgnnsparse_e.so > gpurun_out/sweep2.txt 2>&1
