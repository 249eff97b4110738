#!/bin/bash
# Build tile-shape variants on the GPU box and bench each (development tuning).
# usage: bash tools/sweep.sh "NAME:DEF1,DEF2 ..." workload
mkdir -p gpurun_out /tmp/dcvar
for spec in $1; do
  name=${spec%%:*}; defs=${spec#*:}
  args=""; for d in ${defs//,/ }; do args="$args -D $d"; done
  python paper_conf_ipps_lopez_ortizss13_b200/build.py --out /tmp/dcvar/lib_$name.so $args > /dev/null 2>&1 || { echo "$name build failed"; continue; }
  DC_LIB=/tmp/dcvar/lib_$name.so timeout 300 python bench.py --workload ${2:-sort_u32} --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/sweep_$name.json 2>&1
  python -c "
import json,sys
d=json.loads(open('gpurun_out/sweep_$name.json').read().strip().splitlines()[-1])
k=d.get('kernels', {})
print('$name', round(d['ms_per_step'],4), 'ms', ' '.join(f\"{n}={v['avg_ms']*v['launches_per_step']:.4f}\" for n,v in k.items() if isinstance(v, dict)), 'roof', round(d['roofline']['frac'],3))
" || tail -3 gpurun_out/sweep_$name.json
done
