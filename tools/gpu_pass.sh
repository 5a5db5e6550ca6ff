#!/bin/bash
# usage: tools/gpu_pass.sh TAG  — GPU tests, bench lines for cfg1-4, ncu captures (host loop for frontier kernels)
T=${1:-x}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider 2>&1 | tail -30 > gpurun_out/gpu_tests_$T.log
python bench.py > gpurun_out/bench_${T}_cfg2.json 2> gpurun_out/bench_${T}_cfg2.err
for c in 1 3 4; do
  timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --e2e-steps 1 > gpurun_out/bench_${T}_cfg$c.json 2> gpurun_out/bench_${T}_cfg$c.err
done
if [ -n "$NCU" ]; then
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_pr_gather_apply -s 5 -c 1 -o gpurun_out/prof_${T}_pr python bench.py --steps 1 --warmup 1 --no-cpu --e2e-steps 0 > gpurun_out/ncu_${T}_pr.log 2>&1
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_gather_apply|k_activate" -s 6000 -c 2 -o gpurun_out/prof_${T}_sssp python bench.py --config 3 --steps 1 --warmup 0 --no-cpu --e2e-steps 0 --loop host > gpurun_out/ncu_${T}_sssp.log 2>&1
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_bfs_expand" -s 2 -c 2 -o gpurun_out/prof_${T}_bfs python bench.py --config 1 --steps 1 --warmup 0 --no-cpu --e2e-steps 0 --loop host > gpurun_out/ncu_${T}_bfs.log 2>&1
fi
tail -3 gpurun_out/gpu_tests_$T.log
timeout 600 python -m pytest tests/test_gpu_multirank.py -x -q -m gpu -p no:cacheprovider 2>&1 | tail -30 > gpurun_out/gpu_tests_mr_$T.log
tail -3 gpurun_out/gpu_tests_mr_$T.log
