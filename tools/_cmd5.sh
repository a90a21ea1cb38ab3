mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q --timeout 600 -x > gpurun_out/pytest_gpu5.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu5.txt
timeout 1500 python tools/sweep.py --workload C4 build/libgnnsparse_cur.so > gpurun_out/sweep5.txt 2>&1
timeout 1500 python tools/sweep.py --workload C4 --reorder build/libgnnsparse_cur.so >> gpurun_out/sweep5.txt 2>&1
timeout 1500 python tools/sweep.py --workload C5 --K 256 build/libgnnsparse_cur.so >> gpurun_out/sweep5.txt 2>&1
timeout 1500 python tools/sweep.py --workload C5 --K 256 --reorder build/libgnnsparse_cur.so >> gpurun_out/sweep5.txt 2>&1
