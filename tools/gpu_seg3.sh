#!/bin/bash
# seg kernel v2: parity + bench + hot-table sizes + ncu
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "kernel_variants or pagerank or random or reduced" 2>&1 | tail -3
b() { timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/b_$1.json 2>gpurun_out/b_$1.err; python -c "import json;d=json.load(open('gpurun_out/b_$1.json'));print('$1',d['value'],d['roofline']['avg_launch_us'],d['roofline']['frac'])" || tail -3 gpurun_out/b_$1.err; }
b seg
for k in 24576 40960; do GR_PR_HOTK=$k b seg_k$k; done
if [ -n "$NCU" ]; then
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_pr_seg" -s 10 -c 1 -o gpurun_out/prof_seg2 python bench.py --steps 1 --warmup 1 --no-cpu --e2e-steps 0 > gpurun_out/ncu_seg2.log 2>&1
fi
