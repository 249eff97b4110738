#!/bin/bash
mkdir -p gpurun_out/r02c9
O=gpurun_out/r02c9
for v in default m4_320x79 m4_384x67 m4_448x57 m4_512x49; do
  if [ $v = default ]; then L=""; else L="DC_LIB=variants/$v.so"; fi
  env $L timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_$v.json 2>&1
done
for v in m4_448x57 m4_320x79; do
  DC_LIB=variants/$v.so timeout 600 python tools/variant_check.py > $O/check_$v.txt 2>&1
done
du -sh $O
