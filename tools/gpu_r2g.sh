#!/bin/bash
# round 2: partitioned device-side exchange (sim ranks + two processes), sorted layouts, detail, full suite
T=${1:-r2g}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_multirank.py tests/test_gpu_multiprocess.py -m gpu -x -q --timeout 300 > gpurun_out/${T}_part.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_part.log
timeout 900 python -m pytest tests/test_gpu_sorted.py tests/test_gpu_parity.py -k "sorted or generator or detail" -m gpu -x -q --timeout 300 > gpurun_out/${T}_sorted.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_sorted.log
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_programs.py tests/test_gpu_fullsize.py -m gpu -q --timeout 600 > gpurun_out/${T}_rest.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_rest.log
timeout 300 python bench.py --steps 10 --warmup 3 --e2e-steps 1 > gpurun_out/${T}_cfg2.json 2> gpurun_out/${T}_cfg2.err
GR_PR_PHASES=1 timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > /dev/null 2> gpurun_out/${T}_cfg2_phases.err
ls -la gpurun_out | grep $T
