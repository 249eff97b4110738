#!/bin/bash
mkdir -p gpurun_out/r02c10
O=gpurun_out/r02c10
DC_SWEEP_SIZES=23,24,26,28 timeout 1200 python tools/planner_sweep.py u32_kv > $O/sweep_kv_default.jsonl 2>&1
DC_LIB=variants/kv_256x25.so DC_SWEEP_SIZES=23,24,26,28 timeout 1200 python tools/planner_sweep.py u32_kv > $O/sweep_kv_256x25.jsonl 2>&1
du -sh $O
