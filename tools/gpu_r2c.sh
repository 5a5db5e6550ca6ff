#!/bin/bash
# round 2: programs in every mode, dense gating A/B, PR loop phase split, gather microbench
T=${1:-r2c}
mkdir -p gpurun_out
timeout 600 ./tools/gpaths > gpurun_out/${T}_gpaths.txt 2>&1
GR_PR_PHASES=1 timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/${T}_cfg2_phases.json 2> gpurun_out/${T}_cfg2_phases.err
timeout 1500 python -m pytest tests/test_gpu_programs.py -m gpu -x -q > gpurun_out/${T}_programs.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_programs.log
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -m gpu -x -q > gpurun_out/${T}_parity.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_parity.log
for gt in 0 1; do
  GR_GATE=$gt timeout 600 python bench.py --config 4 --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/${T}_cfg4_g$gt.json 2> /dev/null
  GR_GATE=$gt timeout 600 python bench.py --config 1 --algo sssp --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/${T}_cfg1sssp_g$gt.json 2> /dev/null
  GR_GATE=$gt timeout 600 python bench.py --config 2 --algo pagerank_delta --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/${T}_f2_g$gt.json 2> /dev/null
done
ls -la gpurun_out | grep $T
