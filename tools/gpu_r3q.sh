#!/bin/bash
# changed list carrying the activation range (GR_C_RANGE) A/B on cfg3; record tests
T=${1:-r3q}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
tail -n 2 gpurun_out/${T}_tests.log
for v in 1 0 1 0; do
  GR_C_RANGE=$v timeout 300 python tools/phase_prof.py 3 sssp 1 > gpurun_out/${T}_cfg3_c$v.txt 2>&1
  echo "crange=$v"; tail -n 1 gpurun_out/${T}_cfg3_c$v.txt
done
