#!/bin/bash
mkdir -p gpurun_out/r02c11
O=gpurun_out/r02c11
for v in default m4_960x27 m4_896x29 default; do
  if [ $v = default ]; then L=""; else L="DC_LIB=variants/$v.so"; fi
  env $L timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_$v.json 2>&1
done
for v in m4_960x27 m4_896x29; do
  DC_LIB=variants/$v.so timeout 600 python tools/variant_check.py > $O/check_$v.txt 2>&1
done
du -sh $O
