#!/bin/bash
# time frontier configs with alternative in-tree builds (variants/*.so via GR_LIB)
cd "$(dirname "$0")/.."
python -m pytest tests/test_gpu_parity.py -x -q -k "random or hubs or reduced" > gpurun_out/gpu_tests.txt 2>&1
for lib in default variants/libgr_minb4.so variants/libgr_minb2.so; do
  for c in 3 4 1; do
    tag=$(basename $lib .so)_cfg$c
    if [ "$lib" = default ]; then L=""; else L="$PWD/$lib"; fi
    GR_LIB=$L timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/var_$tag.json 2>/dev/null
  done
done
