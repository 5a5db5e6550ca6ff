#!/bin/bash
# PageRank seg kernel: parity, bench lines vs pipe/warphot, hot-table sweep, ncu
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "kernel_variants or pr_ or pagerank or random" 2>&1 | tail -15 > gpurun_out/seg_tests.log
cat gpurun_out/seg_tests.log | tail -3
for v in warphot pipe seg; do
  GR_PR_KERNEL=$v timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/bench_seg_$v.json 2> gpurun_out/bench_seg_$v.err
  python -c "import json;d=json.load(open('gpurun_out/bench_seg_$v.json'));print('$v',d['value'],d['roofline']['avg_launch_us'],d['roofline']['frac'])" || tail -5 gpurun_out/bench_seg_$v.err
done
for k in 16384 24576 32768 49152 57344; do
  GR_PR_HOTK=$k GR_PR_KERNEL=seg timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/bench_seg_k$k.json 2> /dev/null
  python -c "import json;d=json.load(open('gpurun_out/bench_seg_k$k.json'));print('seg K=$k',d['value'],d['roofline']['avg_launch_us'],d['roofline']['frac'])"
done
if [ -n "$NCU" ]; then
GR_PR_KERNEL=seg timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_pr_seg" -s 10 -c 1 -o gpurun_out/prof_seg python bench.py --steps 1 --warmup 1 --no-cpu --e2e-steps 0 > gpurun_out/ncu_seg.log 2>&1
fi
