#!/bin/bash
mkdir -p gpurun_out/r02c15
O=gpurun_out/r02c15
timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_default.json 2>&1
timeout 300 python bench.py --workload sort_kv --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_kv.json 2>&1
timeout 300 python bench.py --workload sort_u32_small --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_small.json 2>&1
timeout 1800 python -m pytest -x -q tests/test_gpu_parity.py > $O/pytest_parity.txt 2>&1
