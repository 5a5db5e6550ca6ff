#!/bin/bash
# round 2: detail parity, e2e breakdown, then cfg5 at scale (s30 by default): GPU-generated sorted
# layout, one direction borrowed in place, streamed PageRank x30 and BFS
T=${1:-r2j}
mkdir -p gpurun_out
free -g > gpurun_out/${T}_mem.txt; nproc >> gpurun_out/${T}_mem.txt
timeout 600 python -m pytest tests/test_gpu_parity.py -k "detail" -m gpu -q -rf --tb=short --timeout 240 > gpurun_out/${T}_detail.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_detail.log
timeout 300 python tools/e2e_breakdown.py 2 > /dev/null 2> gpurun_out/${T}_e2e_breakdown.txt
GR_TIMING=1 timeout 1500 python bench.py --config 5 --scale ${SCALE:-30} --layout sorted --steps 1 --warmup 1 > gpurun_out/${T}_cfg5_pr.json 2> gpurun_out/${T}_cfg5_pr.err
free -g >> gpurun_out/${T}_mem.txt
GR_TIMING=1 timeout 900 python bench.py --config 5 --scale ${SCALE:-30} --layout sorted --algo bfs --steps 2 --warmup 1 > gpurun_out/${T}_cfg5_bfs.json 2> gpurun_out/${T}_cfg5_bfs.err
ls -la gpurun_out | grep $T
