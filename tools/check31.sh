#!/bin/bash
# Values-only NK4: max-subarray parity tests, bench, ncu of nk4.
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "maxsub or generic or smoke" > gpurun_out/pytest_ms.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_ms.txt
for i in 1 2; do timeout 300 python bench.py --workload maxsub --no-cpu-baseline > gpurun_out/bench_maxsub_$i.json 2> gpurun_out/bench_maxsub_$i.err; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk4_maxsub -s 3 -c 1 -o gpurun_out/prof_nk4 python bench.py --workload maxsub --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu4.txt 2>&1
