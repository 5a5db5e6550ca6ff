#!/bin/bash
# next-row measurements: tolerance PageRank on cfg2, streamed BFS on the cfg5 shape, dense CC gather ncu
cd "$(dirname "$0")/.."
timeout 900 python bench.py --config 2 --algo pagerank_delta --tolerance 1e-4 --steps 3 --warmup 3 --e2e-steps 1 > gpurun_out/f2_cfg2_prdelta.json 2> gpurun_out/f2_cfg2_prdelta.err
timeout 900 python bench.py --config 5 --scale 26 --algo bfs --steps 2 --warmup 3 --e2e-steps 0 --no-cpu > gpurun_out/f1_cfg5s26_bfs.json 2> gpurun_out/f1_cfg5s26_bfs.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather_apply --launch-skip 1 --launch-count 1 -o gpurun_out/ncu_cc_dense -f python bench.py --config 4 --loop host --steps 1 --warmup 0 --e2e-steps 0 --no-cpu > gpurun_out/ncu_cc_dense.log 2>&1
ls -la gpurun_out | tail -5
