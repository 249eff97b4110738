#!/bin/bash
mkdir -p gpurun_out/r02c2
O=gpurun_out/r02c2
timeout 600 python bench.py > $O/bench_default.json 2> $O/bench_default.err
timeout 300 python bench.py --workload maxsub --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_maxsub.json 2>&1
timeout 300 python bench.py --workload sum --steps 10 --warmup 3 > $O/bench_sum.json 2>&1
for v in nk1_256x97 nk1_384x65 nk1_320x77; do
  DC_LIB=variants/$v.so timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_$v.json 2>&1
  DC_LIB=variants/$v.so timeout 600 python tools/variant_check.py > $O/check_$v.txt 2>&1
done
timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_base_again.json 2>&1
timeout 600 python bench.py --impl reference > $O/bench_reference.json 2>&1
