#!/bin/bash
# round profile refresh, summarised on the box (the ncu reports exceed gpurun's copy-back limit)
bash tools/profile_round.sh > /dev/null 2>&1
python tools/summarize_profiles.py r01 > gpurun_out/summarize.txt 2>&1
mkdir -p gpurun_out/profiles_copy
cp -r profiles/* gpurun_out/profiles_copy/
mkdir -p gpurun_out/reps_keep
mv gpurun_out/prof_nk3.ncu-rep gpurun_out/reps_keep/ 2>/dev/null
rm -f gpurun_out/*.ncu-rep
du -sh gpurun_out
