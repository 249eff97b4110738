#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.txt 2>&1
timeout 300 python bench.py --workload sort_kv --no-cpu-baseline > gpurun_out/bench_kv.json 2>&1
timeout 300 python bench.py --workload sort_kv --dist few --no-cpu-baseline --no-e2e > gpurun_out/bench_kv_few.json 2>&1
