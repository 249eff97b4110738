#!/bin/bash
bash tools/sweep.sh "base:DC_STABLE_NT1=512 n256i33:DC_STABLE_NT1=256 n512i25:DC_STABLE_IT=25 n512i17:DC_STABLE_IT=17 n1024i17:DC_STABLE_NT1=1024,DC_STABLE_IT=17" sort_kv > gpurun_out/sweep_kv.txt 2>&1
