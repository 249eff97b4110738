#!/bin/bash
mkdir -p gpurun_out/r02c4
O=gpurun_out/r02c4
timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "every_forced_schedule" > $O/pytest_forced.txt 2>&1
timeout 2400 python tools/planner_sweep.py > $O/planner_sweep.jsonl 2> $O/planner_sweep.err
