#!/bin/bash
# persistent PageRank loop: parity, bench (loop vs launches), ncu of the loop kernel
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "kernel_variants or pagerank or random or reduced or repeated" 2>&1 | tail -3
b() { timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/b_$1.json 2>gpurun_out/b_$1.err; python -c "import json;d=json.load(open('gpurun_out/b_$1.json'));print('$1',d['value'],d['ms_per_step'],d['roofline']['avg_launch_us'],d['roofline']['frac'])" || tail -3 gpurun_out/b_$1.err; }
b loop
GR_PR_LOOP=0 b launches
GR_PR_SEG_VAR=9 b loop_var9
if [ -n "$NCU" ]; then
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_pr_seg_loop" -s 2 -c 1 -o gpurun_out/prof_loop python bench.py --steps 1 --warmup 1 --no-cpu --e2e-steps 0 > gpurun_out/ncu_loop.log 2>&1
tail -3 gpurun_out/ncu_loop.log
fi
