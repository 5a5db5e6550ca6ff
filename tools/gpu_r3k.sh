#!/bin/bash
# symmetric graphs: in-records serve the activation; record tests + cfg3 A/B in one box
T=${1:-r3k}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "records or fullsize or sssp" > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
tail -n 3 gpurun_out/${T}_tests.log
for v in "1 1" "1 0" "1 1" "1 0"; do
  set -- $v
  GR_REC=$1 GR_REC_SYM=$2 timeout 300 python tools/phase_prof.py 3 sssp 1 > gpurun_out/${T}_cfg3_sym$2.txt 2>&1
  echo "sym=$2"; tail -n 1 gpurun_out/${T}_cfg3_sym$2.txt
done
timeout 600 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu --other-configs 0 > gpurun_out/${T}_cfg3.json 2> gpurun_out/${T}_cfg3.err
echo "cfg3 bench $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg3.json)"
