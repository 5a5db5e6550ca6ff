#!/bin/bash
# k_pr_seg variant bits (GR_PR_SEG_VAR) x hot-table size (GR_PR_HOTK) on cfg2 PageRank
mkdir -p gpurun_out
b() { timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/b_$1.json 2>gpurun_out/b_$1.err; python -c "import json;d=json.load(open('gpurun_out/b_$1.json'));print('$1',d['value'],d['roofline']['avg_launch_us'],d['roofline']['frac'])" || tail -3 gpurun_out/b_$1.err; }
for v in 8 9 1 13; do for k in 25596 32768 33780 41980; do GR_PR_HOTK=$k GR_PR_SEG_VAR=$v b segvar${v}_k$k; done; done
