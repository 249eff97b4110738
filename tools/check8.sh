#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q -k "host" > gpurun_out/pytest_host.txt 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 600 python bench.py --workload sort_kv --no-cpu-baseline > gpurun_out/bench_kv.json 2> gpurun_out/bench_kv.err
