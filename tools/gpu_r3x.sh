#!/bin/bash
# packed item position from one shuffle (row start - packed offset), no destination-value shuffle for
# DstFree programs: suite + A/B
T=${1:-r3x}
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
tail -n 2 gpurun_out/${T}_tests.log
for v in main prev main prev; do
  if [ $v = main ]; then unset GR_LIB; else export GR_LIB=variants/libgr_$v.so; fi
  for c in 4 3 1; do
    timeout 240 python bench.py --config $c --steps 5 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg${c}_$v.json 2> /dev/null
    echo "cfg$c $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg${c}_$v.json)"
  done
  timeout 240 python bench.py --config 2 --algo cc --steps 5 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg2cc_$v.json 2> /dev/null
  echo "cfg2cc $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg2cc_$v.json)"
done
