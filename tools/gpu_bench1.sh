#!/bin/bash
# round-1 measurement pass: bench lines + ncu launch list + one full capture
set -x
mkdir -p gpurun_out
python bench.py > gpurun_out/bench_cfg2.json 2> gpurun_out/bench_cfg2.err
for c in 1 3 4; do
  timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --e2e-steps 1 > gpurun_out/bench_cfg$c.json 2> gpurun_out/bench_cfg$c.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_cfg2.csv \
   python bench.py --steps 2 --warmup 1 --no-cpu --e2e-steps 0 > gpurun_out/ncu_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_pr_gather_apply -s 5 -c 1 -o gpurun_out/prof_pr_gather \
   python bench.py --steps 1 --warmup 1 --no-cpu --e2e-steps 0 > gpurun_out/ncu_full.log 2>&1
ls -la gpurun_out
