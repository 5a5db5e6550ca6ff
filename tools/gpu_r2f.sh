#!/bin/bash
# round 2: sorted-layout loads + GPU generator tests, trace detail, then cfg5 at scale (s30) streamed PR + BFS
T=${1:-r2f}
mkdir -p gpurun_out
free -g > gpurun_out/${T}_mem.txt; nproc >> gpurun_out/${T}_mem.txt; lscpu | grep "Model name" >> gpurun_out/${T}_mem.txt
timeout 900 python -m pytest tests/test_gpu_sorted.py tests/test_gpu_parity.py -k "sorted or generator or detail" -m gpu -x -q > gpurun_out/${T}_tests.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_tests.log
if grep -q "rc=0" gpurun_out/${T}_tests.log; then
  timeout 1500 python bench.py --config 5 --scale ${SCALE:-30} --layout sorted --steps 1 --warmup 1 > gpurun_out/${T}_cfg5_pr.json 2> gpurun_out/${T}_cfg5_pr.err
  timeout 900 python bench.py --config 5 --scale ${SCALE:-30} --layout sorted --algo bfs --steps 2 --warmup 1 > gpurun_out/${T}_cfg5_bfs.json 2> gpurun_out/${T}_cfg5_bfs.err
fi
ls -la gpurun_out | grep $T
