#!/bin/bash
# final check of the committed build: full GPU suite, smoke, default bench line, config lines
T=${1:-fin}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
tail -n 2 gpurun_out/${T}_tests.log
timeout 120 python __graft_entry__.py > gpurun_out/${T}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${T}_smoke.log; tail -n 1 gpurun_out/${T}_smoke.log
timeout 900 python bench.py > gpurun_out/${T}_cfg2_default.json 2> gpurun_out/${T}_cfg2_default.err
grep -o '"value": [0-9.]*, "unit": "GTEPS", "n_gpus"' gpurun_out/${T}_cfg2_default.json
for c in 1 3 4; do
  timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-cpu --e2e-steps 1 > gpurun_out/${T}_cfg$c.json 2> /dev/null
  echo "cfg$c $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg$c.json)"
done
timeout 300 python bench.py --config 2 --algo cc --steps 5 --warmup 3 --no-cpu --e2e-steps 0 --other-configs 0 > gpurun_out/${T}_cfg2_cc.json 2> /dev/null
echo "cfg2cc $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg2_cc.json)"
