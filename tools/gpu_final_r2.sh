#!/bin/bash
# round 2 final check on the final build: smoke, the whole -m gpu suite (file by file), default bench
T=${1:-fin2}
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_smoke.log
for f in test_gpu_parity test_gpu_programs test_gpu_multirank test_gpu_multiprocess test_gpu_sorted test_gpu_fullsize; do
  timeout 1200 python -m pytest tests/$f.py -m gpu -q -rf --tb=short --timeout 300 > gpurun_out/${T}_$f.log 2>&1
  echo "rc=$?" >> gpurun_out/${T}_$f.log
done
timeout 900 python bench.py > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err
ls -la gpurun_out | grep $T
