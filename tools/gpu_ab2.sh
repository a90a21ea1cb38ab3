#!/bin/bash
# A/B (kernel-only bench) of the pre-session tree vs the current tree on one box, new tests,
# a 2-rank gloo bench smoke (e2e on row shards).
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "run_host or locality" > gpurun_out/pytest12.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest12.txt
for i in 1 2; do
  (cd build/orig_tree && timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu --no-bf16 --no-compare) > gpurun_out/ab_orig_$i.json 2> gpurun_out/ab_orig_$i.err
  timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu --no-bf16 --no-compare > gpurun_out/ab_cur_$i.json 2> gpurun_out/ab_cur_$i.err
done
GNN_BENCH_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --workload C2 --steps 3 --warmup 3 --no-compare --no-bf16 > gpurun_out/bench12_gloo2.json 2> gpurun_out/bench12_gloo2.err
