#!/bin/bash
# round 2: cp.async tiles phase of the PageRank loop (GR_PR_ASYNC) — parity + A/B; multicast probe
T=${1:-r2m}
mkdir -p gpurun_out
./tools/mc_probe > gpurun_out/${T}_mc_probe.txt 2>&1
GR_PR_ASYNC=1 timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -k "pagerank" -m gpu -q -rf --tb=short --timeout 240 > gpurun_out/${T}_parity_async.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_parity_async.log
for rep in 1 2; do
  for a in 0 1; do
    GR_PR_ASYNC=$a timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --e2e-steps 0 --other-configs 0 > gpurun_out/${T}_cfg2_a${a}_$rep.json 2> /dev/null
  done
done
GR_PR_ASYNC=1 GR_PR_PHASES=1 timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --other-configs 0 > /dev/null 2> gpurun_out/${T}_phases_async.err
ls -la gpurun_out | grep $T
