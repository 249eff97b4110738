#!/bin/bash
mkdir -p gpurun_out/r02c12
O=gpurun_out/r02c12
timeout 2400 python tools/planner_sweep.py u32,f32 > $O/planner_sweep_u32_f32.jsonl 2> $O/planner_sweep.err
timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "two_level or forced or full_size" > $O/pytest_two.txt 2>&1
du -sh $O
