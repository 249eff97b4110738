#!/bin/bash
# Round measurement: default bench line, every bench workload, ncu launch list
# of the default bench command, ncu --set full of the top kernels.
mkdir -p gpurun_out
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
for w in sort_kv sort_u32_small maxsub sum; do
  timeout 300 python bench.py --workload $w --steps 10 --warmup 3 > gpurun_out/bench_$w.json 2>&1
done
for d in sorted reverse few; do
  timeout 300 python bench.py --dist $d --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_sort_u32_$d.json 2>&1
done
timeout 300 python bench.py --workload sort_kv --dist few --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_sort_kv_few.json 2>&1
timeout 120 python tools/pcie_probe.py > gpurun_out/pcie_probe.json 2>&1
timeout 300 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_reference.json 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk3_merge4 -s 20 -c 1 \
  -o gpurun_out/prof_nk3 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk1_blocksort -s 1 -c 1 \
  -o gpurun_out/prof_nk1 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk2_select4 -s 20 -c 1 \
  -o gpurun_out/prof_nk2 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk3_merge4 -s 20 -c 1 \
  -o gpurun_out/prof_nk3_kv python bench.py --workload sort_kv --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk4_maxsub -s 3 -c 1 \
  -o gpurun_out/prof_nk4 python bench.py --workload maxsub --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk1_blocksort -s 1 -c 1 \
  -o gpurun_out/prof_nk1_kv python bench.py --workload sort_kv --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:breadth_first_reduce -s 3 -c 1 \
  -o gpurun_out/prof_sum python bench.py --workload sum --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ls -la gpurun_out
