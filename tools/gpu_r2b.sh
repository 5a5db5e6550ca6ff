#!/bin/bash
# round 2: user programs in every mode (heat, JIT) + L2 policy A/B on cfg4 / cfg3 / cfg1
T=${1:-r2b}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_programs.py -m gpu -x -q > gpurun_out/${T}_programs.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_programs.log
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -m gpu -x -q > gpurun_out/${T}_parity.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_parity.log
for h in 0 1; do
  for c in 4 3 1; do
    GR_L2HINT=$h timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/${T}_cfg${c}_h$h.json 2> /dev/null
  done
done
ls -la gpurun_out | grep $T
