#!/bin/bash
# GR_PULL_DIV sweep (pull when |C_t| * div > |V|) on cfg1 (BFS)
cd "$(dirname "$0")/.."
python -m pytest tests/test_gpu_parity.py -x -q -k "bfs" > gpurun_out/gpu_tests.txt 2>&1
for c in 1; do
  for d in 4 8 16 32 64 128; do
    GR_PULL_DIV=$d timeout 600 python bench.py --config $c --steps 5 --warmup 3 --e2e-steps 0 --no-cpu > gpurun_out/sweep_cfg${c}_${d}.json 2>/dev/null
  done
done
