#!/bin/bash
# round 2: carried A-list CSC ranges — correctness in every path, then cfg3/cfg4/cfg1 A/B (GR_CARRY)
T=${1:-r2k}
mkdir -p gpurun_out
for f in test_gpu_parity test_gpu_programs test_gpu_multirank test_gpu_multiprocess; do
  timeout 900 python -m pytest tests/$f.py -m gpu -q -rf --tb=short --timeout 240 > gpurun_out/${T}_$f.log 2>&1
  echo "rc=$?" >> gpurun_out/${T}_$f.log
done
for c in 1 0; do
  GR_CARRY=$c timeout 600 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --other-configs 0 > gpurun_out/${T}_cfg3_c$c.json 2> /dev/null
  GR_CARRY=$c timeout 600 python bench.py --config 4 --steps 5 --warmup 3 --no-cpu --e2e-steps 0 --other-configs 0 > gpurun_out/${T}_cfg4_c$c.json 2> /dev/null
  GR_CARRY=$c timeout 600 python bench.py --config 1 --algo sssp --steps 10 --warmup 3 --no-cpu --e2e-steps 0 --other-configs 0 > gpurun_out/${T}_cfg1sssp_c$c.json 2> /dev/null
  GR_CARRY=$c timeout 600 python bench.py --config 1 --steps 10 --warmup 3 --no-cpu --e2e-steps 0 --other-configs 0 > gpurun_out/${T}_cfg1_c$c.json 2> /dev/null
done
ls -la gpurun_out | grep $T
