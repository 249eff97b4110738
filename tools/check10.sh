#!/bin/bash
bash tools/sweep.sh "base:DC_TWO_NT=768 t512i51:DC_TWO_NT=512,DC_TWO_IT=51 t512i51m2:DC_TWO_NT=512,DC_TWO_IT=51,DC_M4_MINB=1" sort_u32 > gpurun_out/sweep_m4.txt 2>&1
