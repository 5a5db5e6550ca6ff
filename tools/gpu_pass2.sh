#!/bin/bash
# tests + PageRank variants + frontier configs (+ optional ncu of the default PR kernel)
T=${1:-x}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider 2>&1 | tail -30 > gpurun_out/gpu_tests_$T.log
for v in rangehot range warphot block; do
  GR_PR_KERNEL=$v timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/bench_${T}_pr_$v.json 2> gpurun_out/bench_${T}_pr_$v.err
done
for c in 1 3 4; do
  timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/bench_${T}_cfg$c.json 2> gpurun_out/bench_${T}_cfg$c.err
done
if [ -n "$NCU" ]; then
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_pr_warp_range|k_pr_fixup" -s 10 -c 2 -o gpurun_out/prof_${T}_pr python bench.py --steps 1 --warmup 1 --no-cpu --e2e-steps 0 > gpurun_out/ncu_${T}_pr.log 2>&1
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file gpurun_out/launches_${T}_cfg2.csv python bench.py --steps 2 --warmup 1 --no-cpu --e2e-steps 0 > /dev/null 2>&1
fi
timeout 600 python -m pytest tests/test_gpu_multirank.py -x -q -m gpu -p no:cacheprovider 2>&1 | tail -30 > gpurun_out/gpu_tests_mr_$T.log
tail -3 gpurun_out/gpu_tests_$T.log gpurun_out/gpu_tests_mr_$T.log
