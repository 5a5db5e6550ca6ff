#!/bin/bash
# session restart: full GPU suite, smoke, cfg3/cfg4 baselines on HEAD
T=${1:-r3a}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
timeout 120 python __graft_entry__.py > gpurun_out/${T}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${T}_smoke.log
for c in 3 4; do
  timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --other-configs 0 > gpurun_out/${T}_cfg$c.json 2> gpurun_out/${T}_cfg$c.err
done
tail -3 gpurun_out/${T}_tests.log gpurun_out/${T}_smoke.log
