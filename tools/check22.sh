#!/bin/bash
mkdir -p gpurun_out /tmp/dcvar
python paper_conf_ipps_lopez_ortizss13_b200/build.py --out /tmp/dcvar/lib_pv2.so -D DC_SEL4_PV=2 > /dev/null 2>&1
DC_LIB=/tmp/dcvar/lib_pv2.so timeout 900 python -m pytest tests -m gpu -x -q -k "two_level or full_size or edge or launch" > gpurun_out/pytest_pv2.txt 2>&1
bash tools/sweep.sh "pv4:DC_SEL4_PV=4 pv2:DC_SEL4_PV=2" sort_u32 > gpurun_out/sweep_pv2.txt 2>&1
bash tools/sweep.sh "pv4:DC_SEL4_PV=4 pv2:DC_SEL4_PV=2" sort_kv >> gpurun_out/sweep_pv2.txt 2>&1
