#!/bin/bash
mkdir -p gpurun_out/r02c5
O=gpurun_out/r02c5
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.txt 2>&1
DC_BENCH_DIST=1 timeout 900 python bench.py --steps 5 --warmup 3 > $O/bench_dist_w1.json 2> $O/bench_dist_w1.err
timeout 600 python bench.py --steps 10 --warmup 3 > $O/bench_default.json 2> $O/bench_default.err
timeout 600 python bench.py --workload sort_kv --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_kv.json 2>&1
timeout 300 python bench.py --workload sort_u32_small --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_small.json 2>&1
timeout 120 python tools/mg_profile.py 4 26 0 > $O/mg_profile_a2a.txt 2>&1
timeout 120 python tools/mg_profile.py 8 26 1 > $O/mg_profile_fused.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"mg_|_ab|merge4|select4" -c 14 \
  -o $O/prof_mg_a2a python tools/mg_profile.py 4 26 0 > $O/ncu_mg_a2a.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"_ab|merge4|select4" -c 10 \
  -o $O/prof_mg_fused python tools/mg_profile.py 8 26 1 > $O/ncu_mg_fused.txt 2>&1
