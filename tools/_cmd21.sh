mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_f3.py -q --timeout 900 -x > gpurun_out/pytest_f3.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_f3.txt
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 > gpurun_out/pytest_gpu21.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu21.txt
