#!/bin/bash
# pull-activation check: GPU parity, then cfg1/cfg3/cfg4 push vs auto
cd "$(dirname "$0")/.."
python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.txt 2>&1
for c in 1 4 3; do
  for d in push auto; do
    timeout 600 python bench.py --config $c --steps 3 --warmup 3 --direction $d --e2e-steps 0 --no-cpu > gpurun_out/pull_cfg${c}_${d}.json 2> gpurun_out/pull_cfg${c}_${d}.err
  done
done
