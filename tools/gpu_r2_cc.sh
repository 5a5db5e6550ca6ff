#!/bin/bash
# round 2: dense-superstep source gating (Selective<>) — parity + cfg4/cfg1 bench + ncu of one dense CC gather
T=${1:-r2cc}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${T}_smi.txt
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/${T}_parity.log 2>&1
echo "parity rc=$?" >> gpurun_out/${T}_parity.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -x -q -k "cfg4 or cfg5" > gpurun_out/${T}_fullsize.log 2>&1
echo "fullsize rc=$?" >> gpurun_out/${T}_fullsize.log
for c in 4 1 3; do
  timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/${T}_cfg$c.json 2> gpurun_out/${T}_cfg$c.err
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather_apply --launch-skip 1 --launch-count 1 -o gpurun_out/${T}_ncu_cc_dense -f python bench.py --config 4 --loop host --steps 1 --warmup 0 --e2e-steps 0 --no-cpu > gpurun_out/${T}_ncu.log 2>&1
ls -la gpurun_out | grep $T
