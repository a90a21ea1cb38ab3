mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 > gpurun_out/pytest_gpu23.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu23.txt
GNN_BENCH_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 2 --workload C2 --xmode overlap --steps 2 --warmup 3 --no-compare --no-bf16 > gpurun_out/bench23_overlap.json 2> gpurun_out/bench23_overlap.err
GNN_BENCH_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29513 bench.py --gpus 2 --workload C2 --xmode allgather --steps 2 --warmup 3 --no-compare --no-bf16 > gpurun_out/bench23_ag.json 2> gpurun_out/bench23_ag.err
