#!/bin/bash
# round 2: cfg5 at s30 streamed BFS under the three in-place policies
T=${1:-r2n}
mkdir -p gpurun_out
for zc in -1 1; do
  timeout 900 python bench.py --config 5 --scale 30 --layout sorted --algo bfs --steps 2 --warmup 1 --zero-copy $zc > gpurun_out/${T}_bfs_zc$zc.json 2> gpurun_out/${T}_bfs_zc$zc.err
done
ls -la gpurun_out | grep $T
