#!/bin/bash
bash tools/sweep.sh "base:DC_TWO_NT_KV=512 n768i11:DC_TWO_NT_KV=768,DC_TWO_IT_KV=11 n1024i11:DC_TWO_NT_KV=1024,DC_TWO_IT_KV=11 n256i33:DC_TWO_NT_KV=256,DC_TWO_IT_KV=33 n640i21:DC_TWO_NT_KV=640,DC_TWO_IT_KV=21" sort_kv > gpurun_out/sweep_kv2.txt 2>&1
