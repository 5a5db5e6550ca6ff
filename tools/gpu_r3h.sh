#!/bin/bash
# records/stamp-direct A/B on cfg3 in one box; ncu of the PageRank loop, TMA vs load path; full suite
T=${1:-r3h}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
tail -n 3 gpurun_out/${T}_tests.log
for v in "1 1" "1 0" "0 0" "1 1" "1 0"; do
  set -- $v
  GR_REC=$1 GR_STAMP_DIRECT=$2 timeout 300 python tools/phase_prof.py 3 sssp 1 > gpurun_out/${T}_cfg3_rec$1_sd$2.txt 2>&1
  echo "rec=$1 sd=$2"; tail -n 2 gpurun_out/${T}_cfg3_rec$1_sd$2.txt
done
for tma in 1 0; do
  GR_PR_TMA=$tma timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_pr_seg_loop -c 1 -o gpurun_out/${T}_pr_tma$tma python tools/run_once.py 2 pagerank auto > gpurun_out/${T}_ncu_tma$tma.log 2>&1
  echo "ncu tma$tma rc=$?"
done
