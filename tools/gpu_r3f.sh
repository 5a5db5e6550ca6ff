#!/bin/bash
# cfg3 phase split: records on / gather-only / off; ncu of a mid-run gather + activate (host loop, records on)
T=${1:-r3f}
mkdir -p gpurun_out
GR_REC=1 timeout 300 python tools/phase_prof.py 3 sssp 2 > gpurun_out/${T}_rec1.txt 2>&1
GR_REC=1 GR_REC_OUT=0 timeout 300 python tools/phase_prof.py 3 sssp 2 > gpurun_out/${T}_rec1_out0.txt 2>&1
GR_REC=0 timeout 300 python tools/phase_prof.py 3 sssp 2 > gpurun_out/${T}_rec0.txt 2>&1
tail -n 2 gpurun_out/${T}_rec*.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_gather_apply|k_activate" -s 10000 -c 2 -o gpurun_out/${T}_sssp python tools/run_once.py 3 sssp host > gpurun_out/${T}_ncu.log 2>&1
echo "ncu rc=$?"
