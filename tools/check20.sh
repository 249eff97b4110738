#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "two_level or full_size or max_size or edge or launch" > gpurun_out/pytest_sel.txt 2>&1
timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e > gpurun_out/bench_u32.json 2>&1
timeout 300 python bench.py --workload sort_kv --steps 10 --no-cpu-baseline --no-e2e > gpurun_out/bench_kv.json 2>&1
