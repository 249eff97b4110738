#!/bin/bash
bash tools/sweep.sh "nsel0:DC_M4_NSEL=0 nsel3:DC_M4_NSEL=3 nsel6:DC_M4_NSEL=6,DC_TWO_NT_FUSED=640 nsel2:DC_M4_NSEL=2,DC_TWO_NT_FUSED=736" sort_u32 > gpurun_out/sweep_nsel.txt 2>&1
