#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.txt 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
bash tools/sweep.sh "nt512:DC_FAST_NT1=512 nt1024:DC_FAST_NT1=1024" sort_u32 > gpurun_out/sweep.txt 2>&1
