#!/bin/bash
bash tools/sweep.sh "base:DC_TWO_NT=768 n832i31:DC_TWO_NT=832,DC_TWO_IT=31 n864i29:DC_TWO_NT=864,DC_TWO_IT=29 n704i37:DC_TWO_NT=704,DC_TWO_IT=37" sort_u32 > gpurun_out/sweep_m4b.txt 2>&1
