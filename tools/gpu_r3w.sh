#!/bin/bash
# ncu of the current frontier kernels: cfg3 mid-run gather + activate (records, stamp-direct), cfg4 ungated dense CC superstep
T=${1:-r3w}
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none -k regex:"k_gather_apply|k_activate" -s 20000 -c 2 -o /tmp/${T}_sssp -f python tools/run_once.py 3 sssp host > gpurun_out/${T}_ncu_sssp.log 2>&1
echo "ncu sssp rc=$?"
timeout 900 ncu --set full --clock-control none -k regex:k_gather_apply -s 2 -c 1 -o /tmp/${T}_cc -f python tools/run_once.py 4 cc host > gpurun_out/${T}_ncu_cc.log 2>&1
echo "ncu cc rc=$?"
python tools/summarize_ncu.py full /tmp/${T}_sssp.ncu-rep gpurun_out/${T}_ncu_sssp.md
python tools/summarize_ncu.py full /tmp/${T}_cc.ncu-rep gpurun_out/${T}_ncu_cc.md
ncu -i /tmp/${T}_sssp.ncu-rep --page raw --csv > gpurun_out/${T}_sssp_raw.csv 2>/dev/null
ncu -i /tmp/${T}_cc.ncu-rep --page raw --csv > gpurun_out/${T}_cc_raw.csv 2>/dev/null
ls -la gpurun_out | grep $T
