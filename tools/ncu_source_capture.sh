# ncu --set full with source of the three hot kernels; source pages exported as csv.gz on the box
mkdir -p gpurun_out/src
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk4_maxsub -c 1 -o /tmp/p_nk4 $B --workload maxsub > gpurun_out/src/ncu_nk4.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk3_merge4 -s 3 -c 1 -o /tmp/p_m4 $B > gpurun_out/src/ncu_m4.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nk1_blocksort -c 1 -o /tmp/p_nk1 $B > gpurun_out/src/ncu_nk1.log 2>&1
for k in nk4 m4 nk1; do
  ncu -i /tmp/p_$k.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/src/$k.source.csv.gz
  ncu -i /tmp/p_$k.ncu-rep --page raw --csv 2>/dev/null | gzip > gpurun_out/src/$k.raw.csv.gz
done
ls -la gpurun_out/src
