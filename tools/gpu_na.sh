#!/bin/bash
mkdir -p gpurun_out
GR_PR_SEG_VAR=9 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "kernel_variants and seg" 2>&1 | tail -1
b() { timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/b_$1.json 2>gpurun_out/b_$1.err; python -c "import json;d=json.load(open('gpurun_out/b_$1.json'));print('$1',d['value'],d['ms_per_step'],d['roofline']['avg_launch_us'],d['roofline']['frac'])" || tail -3 gpurun_out/b_$1.err; }
for v in 1 9 3 11; do GR_PR_SEG_VAR=$v b loop_var$v; done
for k in 24576 40960; do GR_PR_HOTK=$k GR_PR_SEG_VAR=9 b loop_var9_k$k; done
