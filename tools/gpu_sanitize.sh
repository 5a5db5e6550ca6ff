#!/bin/bash
mkdir -p gpurun_out
for i in 1 2 3 4 5 6; do
  timeout 300 python -m pytest tests/test_gpu_parity.py -q -m gpu -p no:cacheprovider -k "variants" 2>&1 | tail -2 >> gpurun_out/san_repeat.txt
done
timeout 900 compute-sanitizer --tool racecheck --racecheck-report hazard python tools/sanitize_pr.py warphot 1 > gpurun_out/san_race.txt 2>&1
timeout 900 compute-sanitizer --tool memcheck python tools/sanitize_pr.py warphot 2 > gpurun_out/san_mem.txt 2>&1
timeout 900 compute-sanitizer --tool initcheck python tools/sanitize_pr.py warphot 2 > gpurun_out/san_init.txt 2>&1
tail -5 gpurun_out/san_*.txt
