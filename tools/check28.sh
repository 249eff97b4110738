#!/bin/bash
bash tools/sweep.sh "base:DC_FAST_IT1=51 i49:DC_FAST_IT1=49 i47:DC_FAST_IT1=47" sort_u32 > gpurun_out/sweep_it1.txt 2>&1
