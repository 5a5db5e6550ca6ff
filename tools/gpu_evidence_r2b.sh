#!/bin/bash
# round-2 (second session) evidence: every config line, reference arm, f-rows, ncu launch list +
# --set full of the PageRank loop and of a dense CC gather superstep, PR phase split
T=${1:-ev5}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
timeout 120 python __graft_entry__.py > gpurun_out/${T}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${T}_smoke.log
free -g > gpurun_out/${T}_box.txt; nproc >> gpurun_out/${T}_box.txt; lscpu | grep "Model name" >> gpurun_out/${T}_box.txt
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv >> gpurun_out/${T}_box.txt
python bench.py > gpurun_out/${T}_cfg2_default.json 2> gpurun_out/${T}_cfg2_default.err
python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/${T}_reference.json 2> /dev/null
# the default line above also carries configs 1, 3, 4 and the cfg5 shape (other_configs); e2e lines of those:
for c in 1 3 4; do
  timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu --e2e-steps 1 > gpurun_out/${T}_cfg$c.json 2> /dev/null
done
timeout 600 python bench.py --config 2 --algo cc --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/${T}_cfg2_cc.json 2> /dev/null
timeout 600 python bench.py --config 2 --algo pagerank_delta --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/${T}_f2.json 2> /dev/null
timeout 900 python bench.py --config 5 --scale 26 --layout coo --mode resident --steps 2 --warmup 3 --e2e-steps 0 --no-cpu > gpurun_out/${T}_f3_s26_resident.json 2> /dev/null
GR_PR_PHASES=1 timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --other-configs 0 > /dev/null 2> gpurun_out/${T}_pr_phases.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${T}_launches_default.csv python bench.py --steps 2 --warmup 1 --no-cpu --e2e-steps 0 --other-configs 0 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_pr_seg_loop -c 1 -o gpurun_out/${T}_pr_loop -f python bench.py --steps 1 --warmup 0 --no-cpu --e2e-steps 0 --other-configs 0 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather_apply --launch-skip 5 --launch-count 1 -o gpurun_out/${T}_cc_dense_gated -f python bench.py --config 4 --loop host --steps 1 --warmup 0 --e2e-steps 0 --no-cpu > /dev/null 2>&1
# summaries on the box (the reports themselves exceed what gpurun copies back)
python tools/summarize_ncu.py full gpurun_out/${T}_pr_loop.ncu-rep gpurun_out/${T}_ncu_pr_loop.md > /dev/null 2>&1
python tools/summarize_ncu.py full gpurun_out/${T}_cc_dense_gated.ncu-rep gpurun_out/${T}_ncu_cc_dense_gated.md > /dev/null 2>&1
python tools/summarize_ncu.py launches gpurun_out/${T}_launches_default.csv gpurun_out/${T}_launches_default.md > /dev/null 2>&1
for r in pr_loop cc_dense_gated; do
  ncu -i gpurun_out/${T}_$r.ncu-rep --page raw --csv > gpurun_out/${T}_${r}_raw.csv 2> /dev/null
  ncu -i gpurun_out/${T}_$r.ncu-rep --page source --csv > gpurun_out/${T}_${r}_source.csv 2> /dev/null
  gzip -f gpurun_out/${T}_${r}_source.csv
  rm -f gpurun_out/${T}_$r.ncu-rep
done
ls -la gpurun_out | grep $T
