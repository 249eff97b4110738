#!/bin/bash
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_variants.py -x -q > gpurun_out/pytest_variants.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q --durations=15 > gpurun_out/pytest_gpu.txt 2>&1
