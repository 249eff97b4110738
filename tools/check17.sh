#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q -k "two_level and not stable" > gpurun_out/pytest_fsel.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_fsel.txt
timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e > gpurun_out/bench_u32.json 2>&1
for d in sorted few; do timeout 300 python bench.py --dist $d --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/bench_$d.json 2>&1; done
