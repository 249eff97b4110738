#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_variants.py -x -q > gpurun_out/pytest_variants.txt 2>&1
timeout 600 python -m pytest tests -m gpu -x -q -k "two_level or launch" > gpurun_out/pytest_two.txt 2>&1
timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e > gpurun_out/bench_u32.json 2>&1
