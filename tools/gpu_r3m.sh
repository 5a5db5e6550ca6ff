#!/bin/bash
# changed-set bitmaps read with weak L1-cached loads after the barrier (was ld.global.cg): parity + benches
T=${1:-r3m}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -x -q > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
tail -n 3 gpurun_out/${T}_tests.log
timeout 600 python bench.py --config 2 --algo cc --steps 5 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg2cc.json 2> /dev/null
echo "cfg2cc $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg2cc.json)"
timeout 600 python bench.py --config 2 --algo pagerank_delta --steps 3 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_f2.json 2> /dev/null
echo "f2 $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_f2.json)"
for c in 4 1 3; do
  timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg$c.json 2> /dev/null
  echo "cfg$c $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg$c.json)"
done
timeout 600 python bench.py --config 1 --algo sssp --steps 5 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg1sssp.json 2> /dev/null
echo "cfg1sssp $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg1sssp.json)"
