#!/bin/bash
# round 2: every GPU test file on its own (names of failures reported), short per-test timeouts
T=${1:-r2h}
mkdir -p gpurun_out
for f in test_gpu_multiprocess test_gpu_multirank test_gpu_sorted test_gpu_programs test_gpu_parity test_gpu_fullsize; do
  timeout 1200 python -m pytest tests/$f.py -m gpu -q -rf --tb=short --timeout 240 > gpurun_out/${T}_$f.log 2>&1
  echo "rc=$?" >> gpurun_out/${T}_$f.log
done
ls -la gpurun_out | grep $T
