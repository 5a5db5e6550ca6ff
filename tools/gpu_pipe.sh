#!/bin/bash
# PageRank pipelined warp tiles vs warphot: parity, bench lines, ncu
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "kernel_variants" 2>&1 | tail -5 > gpurun_out/pipe_tests.log
for v in warphot pipe warphot pipe; do
  GR_PR_KERNEL=$v timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/bench_pipe_$v.json 2> gpurun_out/bench_pipe_$v.err
  python -c "import json;d=json.load(open('gpurun_out/bench_pipe_$v.json'));print('$v',d['value'],d['roofline']['avg_launch_us'],d['roofline']['frac'])"
done
if [ -n "$NCU" ]; then
GR_PR_KERNEL=pipe timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_pr_warp_pipe" -s 10 -c 1 -o gpurun_out/prof_pipe python bench.py --steps 1 --warmup 1 --no-cpu --e2e-steps 0 > gpurun_out/ncu_pipe.log 2>&1
fi
cat gpurun_out/pipe_tests.log
