#!/bin/bash
mkdir -p gpurun_out/r02c6
O=gpurun_out/r02c6
timeout 1500 python tools/planner_sweep.py u32 > $O/planner_sweep_u32.jsonl 2> $O/planner_sweep_u32.err
for v in default ms_vonly ms_vonly_j4; do
  if [ $v = default ]; then L=""; else L="DC_LIB=variants/$v.so"; fi
  env $L timeout 300 python bench.py --workload maxsub --steps 20 --warmup 5 --no-cpu-baseline > $O/bench_maxsub_$v.json 2>&1
done
timeout 900 python -m pytest -x -q tests/test_gpu_variants.py -k values_only > $O/pytest_vonly.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk4_maxsub -s 3 -c 1 \
  -o $O/prof_nk4 python bench.py --workload maxsub --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
DC_LIB=variants/ms_vonly.so timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk4_maxsub -s 3 -c 1 \
  -o $O/prof_nk4_vonly python bench.py --workload maxsub --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none -k regex:"mg_|select4|merge4|_ab" -c 32 \
  -o $O/prof_mg_a2a python tools/mg_profile.py 4 25 0 > $O/ncu_mg_a2a.txt 2>&1
timeout 900 ncu --set full --clock-control none -k regex:"select4|merge4|_ab" -c 12 \
  -o $O/prof_mg_fused python tools/mg_profile.py 8 26 1 > $O/ncu_mg_fused.txt 2>&1
for r in prof_mg_a2a prof_mg_fused; do
  python tools/ncu_summary.py $O/$r.ncu-rep > $O/$r.summary.json 2>&1 && rm -f $O/$r.ncu-rep
done
du -sh $O
