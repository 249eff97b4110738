#!/bin/bash
# Round measurement (run under gpurun): bench lines of every workload and
# distribution, the ncu launch list of the default bench command, ncu --set full
# of the top kernels (summarised on the box into JSON and deleted, so the
# copied-back gpurun_out/ stays under 64 MiB), multi-GPU kernels in loopback.
# Then, here: python tools/summarize_profiles.py <round>
mkdir -p gpurun_out
O=gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -q > $O/pytest_gpu.txt 2>&1
timeout 600 python bench.py > $O/bench_default.json 2> $O/bench_default.err
for w in sort_kv sort_u32_small maxsub sum; do
  timeout 300 python bench.py --workload $w --steps 10 --warmup 3 > $O/bench_$w.json 2>&1
done
for d in sorted reverse few; do
  timeout 300 python bench.py --dist $d --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_sort_u32_$d.json 2>&1
done
timeout 300 python bench.py --workload sort_kv --dist few --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_sort_kv_few.json 2>&1
DC_BENCH_DIST=1 timeout 900 python bench.py --workload sort_u32_2p30 --steps 5 --warmup 3 > $O/bench_dist_w1_2p30.json 2>&1
timeout 120 python tools/pcie_probe.py > $O/pcie_probe.json 2>&1
timeout 600 python bench.py --impl reference > $O/bench_reference.json 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file $O/launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
cap() {   # cap <name> <kernel regex> <skip> <bench args...>
  local name=$1 re=$2 skip=$3; shift 3
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$re -s $skip -c 1 \
    -o $O/$name python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline "$@" > /dev/null 2>&1
  python tools/ncu_summary.py $O/$name.ncu-rep > $O/$name.summary.json 2>&1
  ncu -i $O/$name.ncu-rep --page source --csv 2>/dev/null | gzip -9 > $O/$name.source.csv.gz
  rm -f $O/$name.ncu-rep
}
cap prof_nk3 nk3_merge4 20
cap prof_nk1 nk1_blocksort 1
cap prof_nk2 nk2_select4 20
cap prof_nk3_kv nk3_merge4 20 --workload sort_kv
cap prof_nk1_kv nk1_blocksort 1 --workload sort_kv
cap prof_nk4 nk4_maxsub 3 --workload maxsub --warmup 3
cap prof_sum breadth_first_reduce 3 --workload sum --warmup 3
for m in "a2a 4 25 0 mg_|select4|merge4|_ab 32" "fused 8 26 1 select4|merge4|_ab 12"; do
  set -- $m
  timeout 900 ncu --set full --clock-control none -k regex:"$5" -c $6 \
    -o $O/prof_mg_$1 python tools/mg_profile.py $2 $3 $4 > $O/ncu_mg_$1.txt 2>&1
  python tools/ncu_summary.py $O/prof_mg_$1.ncu-rep > $O/prof_mg_$1.summary.json 2>&1
  rm -f $O/prof_mg_$1.ncu-rep
done
ls -la $O; du -sh $O
