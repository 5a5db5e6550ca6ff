#!/bin/bash
# monotone grid barrier + close_superstep batching + REDUX hitmask: full GPU suite, benches, ncu of a dense CC superstep
T=${1:-r3d}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
tail -n 3 gpurun_out/${T}_tests.log
for c in 3 4 2; do
  timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu --other-configs 0 > gpurun_out/${T}_cfg$c.json 2> gpurun_out/${T}_cfg$c.err
  echo cfg$c; grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg$c.json
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_gather_apply -s 2 -c 1 -o gpurun_out/${T}_cc_dense python tools/run_once.py 4 cc host > gpurun_out/${T}_ncu.log 2>&1
echo "ncu rc=$?"
