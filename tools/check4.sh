#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.txt 2>&1
timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 600 python bench.py --workload sort_kv --no-cpu-baseline --no-e2e > gpurun_out/bench_kv.json 2> gpurun_out/bench_kv.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk3_merge4 -s 20 -c 1 \
  -o gpurun_out/prof_nk3 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
