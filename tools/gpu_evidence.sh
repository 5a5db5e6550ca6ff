#!/bin/bash
# round evidence: default bench line, reference arm, other configs (persistent + CUDA-graph loops),
# streamed cfg5 shape, f-rows, ncu launch list of the default bench, ncu --set full of the PR loop
T=${1:-ev}
mkdir -p gpurun_out
python bench.py > gpurun_out/${T}_cfg2_default.json 2> gpurun_out/${T}_cfg2_default.err
python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/${T}_reference.json 2> /dev/null
for c in 1 3 4; do
  timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --e2e-steps 1 > gpurun_out/${T}_cfg$c.json 2> /dev/null
  timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --loop device > gpurun_out/${T}_cfg${c}_graphloop.json 2> /dev/null
done
timeout 900 python bench.py --config 5 --scale 26 --steps 2 --warmup 3 --e2e-steps 1 > gpurun_out/${T}_cfg5s26_streamed.json 2> /dev/null
timeout 900 python bench.py --config 5 --scale 26 --algo bfs --steps 2 --warmup 3 --e2e-steps 0 --no-cpu > gpurun_out/${T}_f1_cfg5s26_bfs.json 2> /dev/null
timeout 900 python bench.py --config 5 --scale 26 --mode resident --steps 2 --warmup 3 --e2e-steps 0 --no-cpu > gpurun_out/${T}_f3_s26_resident.json 2> /dev/null
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${T}_launches_default.csv python bench.py --steps 2 --warmup 1 --no-cpu --e2e-steps 0 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_pr_seg_loop -c 1 -o gpurun_out/${T}_pr_loop -f python bench.py --steps 1 --warmup 0 --no-cpu --e2e-steps 0 > /dev/null 2>&1
ls -la gpurun_out | grep $T
