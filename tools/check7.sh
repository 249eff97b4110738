#!/bin/bash
mkdir -p gpurun_out
timeout 120 python tools/pcie_probe.py > gpurun_out/pcie.json 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "val or kv or stable or f32 or pairs or two_level" > gpurun_out/pytest_kv.txt 2>&1
timeout 600 python bench.py --workload sort_kv --no-cpu-baseline --no-e2e > gpurun_out/bench_kv.json 2> gpurun_out/bench_kv.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk1_blocksort -s 1 -c 1 \
  -o gpurun_out/prof_nk1_kv python bench.py --workload sort_kv --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
