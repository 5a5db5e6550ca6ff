#!/bin/bash
# PageRank hot-table size sweep on the current loop (GR_PR_HOTK), L1 = what the table leaves
T=${1:-r3u}
mkdir -p gpurun_out
for k in 32768 24576 28672 36864 32768 24576 28672 36864; do
  GR_PR_HOTK=$k timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_k$k.json 2> /dev/null
  echo "hotk $k $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_k$k.json)"
done
