mkdir -p gpurun_out
timeout 600 python tools/microbench.py > gpurun_out/microbench.json 2> gpurun_out/microbench.err
timeout 900 python -m pytest tests -m gpu -q --timeout 600 -x > gpurun_out/pytest_gpu3.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu3.txt
timeout 1500 python tools/sweep.py --workload C4 --vw8 build/libgnnsparse_a.so build/libgnnsparse_f.so build/libgnnsparse_g.so build/libgnnsparse_h.so build/libgnnsparse_i.so > gpurun_out/sweep3.txt 2>&1
