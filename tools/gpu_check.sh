#!/bin/bash
# GPU-box check used during development: smoke, GPU parity tests, short benches, ncu captures.
set -x
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
for w in sort_u32 sort_kv sort_u32_small; do timeout 300 python bench.py --workload $w --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_$w.json 2>&1; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk1_blocksort -s 1 -c 1 -o gpurun_out/prof_nk1 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu1.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk3_merge -s 20 -c 1 -o gpurun_out/prof_nk3 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu3.txt 2>&1
