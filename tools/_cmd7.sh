mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 > gpurun_out/pytest_gpu7.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu7.txt
timeout 600 python bench.py --workload C3 --steps 20 --warmup 3 > gpurun_out/bench7_c3.json 2> gpurun_out/bench7_c3.err
timeout 900 python bench.py --workload C5 --steps 5 --warmup 3 --no-cpu > gpurun_out/bench7_c5.json 2> gpurun_out/bench7_c5.err
GNN_BENCH_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 3 --warmup 3 --no-compare > gpurun_out/bench7_2rank.json 2> gpurun_out/bench7_2rank.err
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench7_ref.json 2> gpurun_out/bench7_ref.err
