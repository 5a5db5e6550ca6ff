#!/bin/bash
# TMA item stream for the PageRank loop (A/B), records (gather only) + no pre-read activation: suite + benches
T=${1:-r3g}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
tail -n 3 gpurun_out/${T}_tests.log
for tma in 1 0 1 0; do
  GR_PR_TMA=$tma timeout 600 python bench.py --config 2 --steps 10 --warmup 3 --no-cpu --other-configs 0 > gpurun_out/${T}_cfg2_tma$tma.json 2> gpurun_out/${T}_cfg2_tma$tma.err
  echo cfg2 tma$tma; grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg2_tma$tma.json
done
for tma in 1 0; do
  GR_PR_TMA=$tma GR_PR_PHASES=1 timeout 300 python tools/run_once.py 2 pagerank auto > gpurun_out/${T}_phases_tma$tma.txt 2>&1
  tail -n 2 gpurun_out/${T}_phases_tma$tma.txt
done
for c in 3 4; do
  timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --other-configs 0 > gpurun_out/${T}_cfg$c.json 2> gpurun_out/${T}_cfg$c.err
  echo cfg$c; grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg$c.json
done
