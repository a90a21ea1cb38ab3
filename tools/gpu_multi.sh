#!/bin/bash
# run_host_multi session: full GPU tests, bench, compute-sanitizer on small cases.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider > gpurun_out/pytest_multi.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_multi.txt
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_multi.json 2> gpurun_out/bench_multi.err; echo "rc=$?" >> gpurun_out/bench_multi.err
timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "c1_tiny or c2_cora or empty_rows or hub_row or run_host_pipelined_pieces or multi_widths or leading" > gpurun_out/sanitizer_memcheck.txt 2>&1; echo "rc=$?" >> gpurun_out/sanitizer_memcheck.txt
timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "c1_tiny or c2_cora or empty_rows or hub_row" > gpurun_out/sanitizer_racecheck.txt 2>&1; echo "rc=$?" >> gpurun_out/sanitizer_racecheck.txt
timeout 900 compute-sanitizer --tool synccheck --error-exitcode 9 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "c1_tiny or c2_cora or empty_rows" > gpurun_out/sanitizer_synccheck.txt 2>&1; echo "rc=$?" >> gpurun_out/sanitizer_synccheck.txt
