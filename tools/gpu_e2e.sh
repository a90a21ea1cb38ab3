#!/bin/bash
# e2e pipeline session: new run_host tests, then bench e2e at several piece counts.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 600 -p no:cacheprovider -k "run_host" > gpurun_out/pytest_runhost.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_runhost.txt
for P in 1 8 16 32; do
  GNN_HOST_PIECES=$P timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-bf16 --no-compare > gpurun_out/bench_e2e_p$P.json 2> gpurun_out/bench_e2e_p$P.err
done
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-bf16 --no-compare > gpurun_out/bench_e2e_default.json 2> gpurun_out/bench_e2e_default.err
