#!/bin/bash
# compute-sanitizer over tools/sanitize_run.py (small sizes; memcheck also at >= 2^23).
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  extra=""
  [ "$tool" = "memcheck" ] && extra="--large"
  timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py $extra \
    > gpurun_out/sanitize_$tool.txt 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|sanitize_run ok' gpurun_out/sanitize_$tool.txt | tr '\n' ' ')"
done
