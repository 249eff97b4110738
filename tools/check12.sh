#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "small or graph or fused or 2pow20 or oracle" > gpurun_out/pytest_small.txt 2>&1
timeout 300 python bench.py --workload sort_u32_small --steps 20 --no-cpu-baseline > gpurun_out/bench_small.json 2>&1
