#!/bin/bash
# next-group L1 prefetch (implicit / dense supersteps) A/B; parity of the gather
T=${1:-r3p}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
tail -n 2 gpurun_out/${T}_tests.log
for v in main nonext main nonext; do
  if [ $v = main ]; then unset GR_LIB; else export GR_LIB=variants/libgr_$v.so; fi
  timeout 600 python bench.py --config 4 --steps 5 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg4_$v.json 2> /dev/null
  echo "cfg4 $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg4_$v.json)"
  timeout 600 python bench.py --config 2 --algo cc --steps 5 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg2cc_$v.json 2> /dev/null
  echo "cfg2cc $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg2cc_$v.json)"
  timeout 600 python bench.py --config 1 --steps 5 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg1_$v.json 2> /dev/null
  echo "cfg1 $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg1_$v.json)"
done
