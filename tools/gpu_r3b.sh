#!/bin/bash
# locality-window dense gather: parity + cfg4 A/B
T=${1:-r3b}
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "window or dense_tile" > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
for w in 1 0 1 0; do
  GR_DENSE_WIN=$w timeout 600 python bench.py --config 4 --steps 5 --warmup 3 --no-cpu --other-configs 0 > gpurun_out/${T}_cfg4_w$w.json 2> gpurun_out/${T}_cfg4_w$w.err
  grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg4_w$w.json
done
