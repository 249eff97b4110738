#!/bin/bash
mkdir -p gpurun_out/r02c8
O=gpurun_out/r02c8
timeout 1500 python -m pytest -x -q tests/test_gpu_native_mg.py > $O/pytest_mg.txt 2>&1
timeout 1200 python -m pytest -x -q tests/test_gpu_variants.py > $O/pytest_variants.txt 2>&1
timeout 900 ncu --set full --clock-control none -k regex:"mg_|select4|merge4|_ab" -c 32 \
  -o $O/prof_mg_a2a python tools/mg_profile.py 4 25 0 > $O/ncu_mg_a2a.txt 2>&1
timeout 900 ncu --set full --clock-control none -k regex:"mg_" -c 40 \
  -o $O/prof_mg_g8 python tools/mg_profile.py 8 26 0 > $O/ncu_mg_g8.txt 2>&1
for r in prof_mg_a2a prof_mg_g8; do
  python tools/ncu_summary.py $O/$r.ncu-rep > $O/$r.summary.json 2>&1 && rm -f $O/$r.ncu-rep
done
timeout 2400 bash tools/sanitize.sh > $O/sanitize_summary.txt 2>&1
mkdir -p $O/san && cp gpurun_out/sanitize_*.txt $O/san/ 2>/dev/null
du -sh $O
