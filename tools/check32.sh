#!/bin/bash
# Max-subarray parity (default + values-only variant) and bench.
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_variants.py -m gpu -x -q -k "maxsub" > gpurun_out/pytest_ms.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_ms.txt
timeout 300 python bench.py --workload maxsub --no-cpu-baseline > gpurun_out/bench_maxsub_1.json 2> gpurun_out/bench_maxsub_1.err
