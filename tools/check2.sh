#!/bin/bash
# Development check: GPU tests, default bench, NK1 ncu capture.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.txt 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk1_ -s 1 -c 1 \
  -o gpurun_out/prof_nk1 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu1.txt 2>&1
