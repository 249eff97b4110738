#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "two_level or full_size or max_size or edge or launch" > gpurun_out/pytest_fit.txt 2>&1
bash tools/sweep.sh "fit:DC_TWO_FIT=1 nofit:DC_TWO_FIT=0" sort_u32 > gpurun_out/sweep_fit.txt 2>&1
