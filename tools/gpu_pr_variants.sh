#!/bin/bash
# PageRank gather variants: parity + cfg2 bench line + ncu capture for each
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider 2>&1 | tail -30 > gpurun_out/gpu_tests_pv.log
for v in warp warphot block blockhot; do
  GR_PR_KERNEL=$v timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/bench_pv_$v.json 2> gpurun_out/bench_pv_$v.err
done
for v in warp warphot; do
  GR_PR_KERNEL=$v timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_pr_warp|k_pr_fixup" -s 10 -c 2 -o gpurun_out/prof_pv_$v python bench.py --steps 1 --warmup 1 --no-cpu --e2e-steps 0 > gpurun_out/ncu_pv_$v.log 2>&1
done
tail -3 gpurun_out/gpu_tests_pv.log
