#!/bin/bash
# vertex records (GR_REC) + launch bounds: full GPU suite, cfg3 A/B, cfg4, cfg1
T=${1:-r3e}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
tail -n 3 gpurun_out/${T}_tests.log
for r in 1 0; do
  GR_REC=$r timeout 600 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu --other-configs 0 > gpurun_out/${T}_cfg3_rec$r.json 2> gpurun_out/${T}_cfg3_rec$r.err
  echo cfg3 rec$r; grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg3_rec$r.json
done
GR_REC=1 timeout 300 python tools/phase_prof.py 3 sssp 2 > gpurun_out/${T}_cfg3_phases.txt 2>&1; cat gpurun_out/${T}_cfg3_phases.txt
for c in 4 1; do
  timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu --other-configs 0 > gpurun_out/${T}_cfg$c.json 2> gpurun_out/${T}_cfg$c.err
  echo cfg$c; grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg$c.json
done
