#!/bin/bash
# round 2: handle-cache build validation + multicast probe
T=${1:-r2l}
mkdir -p gpurun_out
./tools/mc_probe > gpurun_out/${T}_mc_probe.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_smoke.log
for f in test_gpu_parity test_gpu_multiprocess test_gpu_multirank; do
  timeout 900 python -m pytest tests/$f.py -m gpu -q -rf --tb=short --timeout 240 > gpurun_out/${T}_$f.log 2>&1
  echo "rc=$?" >> gpurun_out/${T}_$f.log
done
timeout 300 python tools/e2e_breakdown.py 2 > /dev/null 2> gpurun_out/${T}_e2e.txt
timeout 600 python bench.py --steps 10 --warmup 3 --other-configs 0 > gpurun_out/${T}_cfg2.json 2> /dev/null
ls -la gpurun_out | grep $T
