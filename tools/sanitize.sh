#!/bin/bash
# compute-sanitizer over tools/sanitize_run.py (small sizes; memcheck also at >= 2^23).
mkdir -p gpurun_out
# initcheck does not see TMA bulk stores as initialising global memory: run it on
# a variant whose tiles leave through plain stores (same kernels otherwise).
python paper_conf_ipps_lopez_ortizss13_b200/build.py --out /tmp/dc_notma.so -D DC_NO_TMA_STORE > /dev/null
for tool in memcheck racecheck synccheck initcheck; do
  extra=""
  [ "$tool" = "memcheck" ] && extra="--large"
  lib=""
  [ "$tool" = "initcheck" ] && lib="DC_LIB=/tmp/dc_notma.so"
  env $lib timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py $extra \
    > gpurun_out/sanitize_$tool.txt 2>&1
  echo "$tool rc=$? $(grep -E 'SUMMARY|sanitize_run ok' gpurun_out/sanitize_$tool.txt | tr '\n' ' ')"
done
