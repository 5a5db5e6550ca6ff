#!/bin/bash
# seg kernel: no-allocate cold gathers, hot-table sizes
mkdir -p gpurun_out
b() { timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/b_$1.json 2>/dev/null; python -c "import json;d=json.load(open('gpurun_out/b_$1.json'));print('$1',d['value'],d['roofline']['avg_launch_us'],d['roofline']['frac'])"; }
b seg
for k in 24576 32768 40960; do
  GR_LIB=$PWD/variants/libgr_segna.so GR_PR_HOTK=$k b segna_k$k
done
b seg
