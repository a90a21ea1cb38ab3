mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_f3.py -q --timeout 900 > gpurun_out/pytest_f3b.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_f3b.txt
timeout 1200 python tools/train_gcn.py --workload C4 --hidden 32,128,256 --steps 10 > gpurun_out/train_c4.txt 2>&1
timeout 1200 python tools/train_gcn.py --workload C4 --reorder --hidden 32,128,256 --steps 10 > gpurun_out/train_c4gcr.txt 2>&1
timeout 600 python tools/train_gcn.py --workload C2 --hidden 32,128,256 --features 128 --classes 10 --steps 20 > gpurun_out/train_c2.txt 2>&1
