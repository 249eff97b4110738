#!/bin/bash
# r02 call 3: full GPU suite after the Pass4 refactor + 4-way G-way merge,
# smoke, dist bench at world 1 (both exchange modes), default bench.
mkdir -p gpurun_out/r02c3
O=gpurun_out/r02c3
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.txt 2>&1
DC_BENCH_DIST=1 timeout 900 python bench.py --steps 5 --warmup 3 > $O/bench_dist_w1.json 2> $O/bench_dist_w1.err
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_default.json 2> $O/bench_default.err
