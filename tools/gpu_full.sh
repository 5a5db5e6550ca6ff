#!/bin/bash
# full round measurement: default bench line, reference arm, streamed cfg5-shape, loop comparison, ncu launch list
T=${1:-full}
mkdir -p gpurun_out
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/clocks_$T.txt
python bench.py > gpurun_out/bench_${T}_default.json 2> gpurun_out/bench_${T}_default.err
python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_${T}_reference.json 2> gpurun_out/bench_${T}_reference.err
timeout 900 python bench.py --config 5 --scale 26 --steps 2 --warmup 3 --e2e-steps 1 > gpurun_out/bench_${T}_cfg5s26.json 2> gpurun_out/bench_${T}_cfg5s26.err
for c in 1 3 4; do
  timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --e2e-steps 1 > gpurun_out/bench_${T}_cfg$c.json 2> gpurun_out/bench_${T}_cfg$c.err
  timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --loop device > gpurun_out/bench_${T}_cfg${c}_graph.json 2> /dev/null
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_${T}_default.csv python bench.py --steps 2 --warmup 1 --no-cpu --e2e-steps 0 > /dev/null 2>&1
ls -la gpurun_out | tail -30
