#!/bin/bash
# with the small shared footprint: activation records / symmetric record reuse A/B on cfg3 (env only)
T=${1:-r3t}
mkdir -p gpurun_out
for v in base out sym base out sym; do
  unset GR_REC_OUT GR_REC_SYM
  [ $v = out ] && export GR_REC_OUT=1
  [ $v = sym ] && export GR_REC_SYM=1
  timeout 600 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg3_$v.json 2> /dev/null
  echo "cfg3 $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg3_$v.json)"
done
