#!/bin/bash
# persisting-L2 access-policy window over the vertex values (GR_L2_PERSIST) A/B: cfg4, cfg3, cfg2 cc
T=${1:-r3l}
mkdir -p gpurun_out
for p in 0 1 0 1; do
  for c in 4 3; do
    GR_L2_PERSIST=$p timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg${c}_p$p.json 2> gpurun_out/${T}_cfg${c}_p$p.err
    echo "cfg$c p$p $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg${c}_p$p.json) $(grep -h 'L2 persisting' gpurun_out/${T}_cfg${c}_p$p.err | head -1)"
  done
done
