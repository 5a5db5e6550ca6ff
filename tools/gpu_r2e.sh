#!/bin/bash
# round 2: adaptive gating + device-side count exchange: full GPU suite, timings
T=${1:-r2e}
mkdir -p gpurun_out
timeout 2400 python -m pytest tests/ -m gpu -x -q --deselect tests/test_gpu_fullsize.py > gpurun_out/${T}_gpu.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_gpu.log
for rep in 1 2; do
  timeout 600 python bench.py --config 4 --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/${T}_cfg4_$rep.json 2> /dev/null
  timeout 600 python bench.py --config 2 --algo cc --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/${T}_cfg2cc_$rep.json 2> /dev/null
  timeout 600 python bench.py --config 1 --algo sssp --steps 10 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/${T}_cfg1sssp_$rep.json 2> /dev/null
done
timeout 600 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/${T}_cfg3.json 2> /dev/null
timeout 600 python bench.py --steps 10 --warmup 3 --e2e-steps 1 > gpurun_out/${T}_cfg2.json 2> gpurun_out/${T}_cfg2.err
ls -la gpurun_out | grep $T
