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
# The two-level pass kernels (nk2_select4, nk3_merge4: mbarriers, named barriers, TMA) run only
# for n >= 2^23 inside the library; check them in isolation at small sizes (many tiles per CTA).
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo \
  -I include -I paper_conf_ipps_lopez_ortizss13_b200/csrc tools/sort4_check.cu -o /tmp/sort4_check
# the same kernel with named-barrier hand-offs and plain copies (DC_M4_BARRIER_HANDOFF):
# racecheck models bar.arrive / bar.sync, so this isolates the default build's
# reports to the mbarrier / TMA hand-off
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -DDC_M4_BARRIER_HANDOFF=1 \
  -I include -I paper_conf_ipps_lopez_ortizss13_b200/csrc tools/sort4_check.cu -o /tmp/sort4_check_bar
out=gpurun_out/sanitize_sort4_barrier_racecheck.txt
: > $out
for a in "200000 26112 0 0 2" "1000003 26112 1 0 3" "500001 26112 2" "400000 104448 3 0 1"; do
  timeout 900 compute-sanitizer --tool racecheck --print-limit 20 /tmp/sort4_check_bar $a >> $out 2>&1
done
echo "sort4 barrier-handoff racecheck: $(grep -cE 'mismatches' $out) checks, $(grep -E 'RACECHECK SUMMARY' $out | tr '\n' ' ')"
for tool in memcheck racecheck synccheck; do
  out=gpurun_out/sanitize_sort4_$tool.txt
  : > $out
  for a in "200000 26112 0 0 2" "1000003 26112 1 0 3" "500001 26112 2" "400000 104448 3 0 1"; do
    timeout 900 compute-sanitizer --tool $tool --print-limit 20 /tmp/sort4_check $a >> $out 2>&1
  done
  echo "sort4 $tool: $(grep -cE 'mismatches' $out) checks, $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' $out | tr '\n' ' ')"
done
