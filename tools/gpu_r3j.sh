#!/bin/bash
# bits-free ungated dense gather (probe only unchanged vertices) vs reading every bit: suite + A/B
T=${1:-r3j}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
tail -n 3 gpurun_out/${T}_tests.log
for v in base bits base bits; do
  if [ $v = bits ]; then export GR_LIB=variants/libgr_bits.so; else unset GR_LIB; fi
  timeout 600 python bench.py --config 4 --steps 5 --warmup 3 --no-cpu --other-configs 0 > gpurun_out/${T}_cfg4_$v.json 2> gpurun_out/${T}_cfg4_$v.err
  echo "cfg4 $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg4_$v.json)"
  timeout 600 python bench.py --config 2 --algo cc --steps 5 --warmup 3 --no-cpu --other-configs 0 > gpurun_out/${T}_cfg2cc_$v.json 2> gpurun_out/${T}_cfg2cc_$v.err
  echo "cfg2cc $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg2cc_$v.json)"
  timeout 600 python bench.py --config 1 --algo sssp --steps 5 --warmup 3 --no-cpu --other-configs 0 > gpurun_out/${T}_cfg1sssp_$v.json 2> gpurun_out/${T}_cfg1sssp_$v.err
  echo "cfg1sssp $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg1sssp_$v.json)"
done
