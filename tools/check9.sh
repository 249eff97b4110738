#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "two_level or full_size or select or max_size or edge" > gpurun_out/pytest_sel.txt 2>&1
for d in uniform sorted reverse few; do
  timeout 300 python bench.py --dist $d --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/bench_$d.json 2>&1
done
timeout 300 python bench.py --workload sort_kv --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/bench_kv.json 2>&1
