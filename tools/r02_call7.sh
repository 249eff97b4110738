#!/bin/bash
mkdir -p gpurun_out/r02c7
O=gpurun_out/r02c7
timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "maxsub" > $O/pytest_maxsub.txt 2>&1
for v in default ms_tma ms_rows20s3 ms_rows36 ms_rows44 ms_rows28s3; do
  if [ $v = default ]; then L=""; else L="DC_LIB=variants/$v.so"; fi
  env $L timeout 300 python bench.py --workload maxsub --steps 20 --warmup 5 --no-cpu-baseline > $O/bench_maxsub_$v.json 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk4_maxsub -s 3 -c 1 \
  -o $O/prof_nk4_rows python bench.py --workload maxsub --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.txt 2>&1
du -sh $O
