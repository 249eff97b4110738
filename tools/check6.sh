#!/bin/bash
bash tools/sweep.sh "base:DC_MS_P=68 t512p36:DC_MS_TNT=512,DC_MS_P=36 t384p44:DC_MS_TNT=384,DC_MS_P=44 t512p36s3:DC_MS_TNT=512,DC_MS_P=36,DC_MS_S=3,DC_MS_J=1 t256p36s4:DC_MS_P=36,DC_MS_S=4" maxsub > gpurun_out/sweep_ms.txt 2>&1
