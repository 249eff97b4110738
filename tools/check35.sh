#!/bin/bash
# NK4 shape sweep (lane chunk L = DC_MS_P, chains J = DC_MS_J) on the max-subarray bench.
mkdir -p gpurun_out
for v in default j1 j3 j4 p52 p60 p76; do
  if [ $v = default ]; then unset DC_LIB; else export DC_LIB=$PWD/paper_conf_ipps_lopez_ortizss13_b200/libdc_$v.so; fi
  echo -n "$v " >> gpurun_out/sweep_ms.txt
  timeout 120 python bench.py --workload maxsub --no-cpu-baseline --no-e2e --steps 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d['ms_per_step'], d['roofline']['avg_launch_ms'])" >> gpurun_out/sweep_ms.txt
done
