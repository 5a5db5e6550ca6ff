#!/bin/bash
# superstep close by the last CTA to arrive at the end-of-superstep barrier vs barrier / CTA 0 / barrier
T=${1:-r3v}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
tail -n 2 gpurun_out/${T}_tests.log
timeout 120 python __graft_entry__.py > gpurun_out/${T}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${T}_smoke.log; tail -n 1 gpurun_out/${T}_smoke.log
for v in main cta0 main cta0; do
  if [ $v = main ]; then unset GR_LIB; else export GR_LIB=variants/libgr_$v.so; fi
  for c in 3 1 4; do
    timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu --other-configs 0 --e2e-steps 0 > gpurun_out/${T}_cfg${c}_$v.json 2> /dev/null
    echo "cfg$c $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg${c}_$v.json)"
  done
done
