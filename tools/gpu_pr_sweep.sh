#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider 2>&1 | tail -30 > gpurun_out/gpu_tests_sw.log
for cfg in "16384 1024" "16384 768" "24576 1024" "24576 768" "32768 768" "32768 512" "8192 1024"; do
  set -- $cfg
  GR_PR_KERNEL=warphot GR_PR_HOTK=$1 GR_PR_CTA=$2 timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/bench_sw_$1_$2.json 2> gpurun_out/bench_sw_$1_$2.err
done
GR_PR_KERNEL=rangehot timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/bench_sw_rangehot.json 2>/dev/null
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file gpurun_out/launches_sw_cfg2.csv python bench.py --steps 2 --warmup 1 --no-cpu --e2e-steps 0 > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_multirank.py -x -q -m gpu -p no:cacheprovider 2>&1 | tail -5 > gpurun_out/gpu_tests_mr_sw.log
tail -3 gpurun_out/gpu_tests_sw.log gpurun_out/gpu_tests_mr_sw.log
