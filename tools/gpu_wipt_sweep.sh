#!/bin/bash
# warp-tile size x hot-table size sweep for k_pr_warp_hot (cfg2)
cd "$(dirname "$0")/.."
GR_LIB=$PWD/variants/libgr_wipt4.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "pagerank" > gpurun_out/wipt4_tests.txt 2>&1
for k in 16384 24576; do
  GR_PR_HOTK=$k timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/wipt8_$k.json 2>/dev/null
done
for k in 16384 32768 40960 45056; do
  GR_LIB=$PWD/variants/libgr_wipt4.so GR_PR_HOTK=$k timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/wipt4_$k.json 2>/dev/null
done
