#!/bin/bash
# round 2: two real processes (shm transport + cudaIpc), programs, gating A/B (compile-time variants)
T=${1:-r2d}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_multiprocess.py -m gpu -x -q > gpurun_out/${T}_mp.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_mp.log
timeout 900 python -m pytest tests/test_gpu_programs.py -m gpu -x -q > gpurun_out/${T}_programs.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_programs.log
for v in gate nogate; do
  L=""; [ $v = nogate ] && L="variants/libgr_nogate.so"
  for rep in 1 2; do
    GR_LIB=$L timeout 600 python bench.py --config 4 --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/${T}_cfg4_${v}_$rep.json 2> /dev/null
    GR_LIB=$L timeout 600 python bench.py --config 1 --algo sssp --steps 10 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/${T}_cfg1sssp_${v}_$rep.json 2> /dev/null
    GR_LIB=$L timeout 600 python bench.py --config 2 --algo cc --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/${T}_cfg2cc_${v}_$rep.json 2> /dev/null
  done
done
ls -la gpurun_out | grep $T
