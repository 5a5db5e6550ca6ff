#!/bin/bash
# packed gather up to 128 in-edges per lane (GR_PACK_DEG) vs 32: parity + A/B in one box
T=${1:-r3n}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
tail -n 3 gpurun_out/${T}_tests.log
for v in p128 p32 p128 p32; do
  if [ $v = p32 ]; then export GR_LIB=variants/libgr_p32.so; else unset GR_LIB; fi
  for c in 4 3; do
    timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg${c}_$v.json 2> /dev/null
    echo "cfg$c $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg${c}_$v.json)"
  done
  timeout 600 python bench.py --config 2 --algo cc --steps 5 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg2cc_$v.json 2> /dev/null
  echo "cfg2cc $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg2cc_$v.json)"
  timeout 600 python bench.py --config 1 --algo sssp --steps 5 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg1sssp_$v.json 2> /dev/null
  echo "cfg1sssp $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg1sssp_$v.json)"
done
