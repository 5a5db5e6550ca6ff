#!/bin/bash
# grid-barrier variants, per-phase split of cfg3/cfg4, window A/B
T=${1:-r3c}
mkdir -p gpurun_out
./tools/gsb > gpurun_out/${T}_gsb.txt 2>&1
timeout 300 python tools/phase_prof.py 3 sssp 2 > gpurun_out/${T}_cfg3_phases.txt 2>&1
for w in 0 1; do GR_DENSE_WIN=$w timeout 300 python tools/phase_prof.py 4 cc 3 > gpurun_out/${T}_cfg4_w${w}_phases.txt 2>&1; done
timeout 600 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu --other-configs 0 > gpurun_out/${T}_cfg3.json 2> gpurun_out/${T}_cfg3.err
grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg3.json
cat gpurun_out/${T}_gsb.txt gpurun_out/${T}_*phases.txt
