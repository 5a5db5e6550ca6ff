#!/bin/bash
# resident CTAs per SM for the 32-bit loops now that shared memory is small: 4 (main) / 5 / 6
T=${1:-r3s}
mkdir -p gpurun_out
for v in main c5 c6 main c5 c6; do
  if [ $v = main ]; then unset GR_LIB GR_PERSIST_CTAS_PER_SM; else export GR_LIB=variants/libgr_$v.so GR_PERSIST_CTAS_PER_SM=${v#c}; fi
  for c in 4 3 1; do
    timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg${c}_$v.json 2> /dev/null
    echo "cfg$c $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg${c}_$v.json)"
  done
  timeout 600 python bench.py --config 2 --algo cc --steps 5 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg2cc_$v.json 2> /dev/null
  echo "cfg2cc $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg2cc_$v.json)"
done
