#!/bin/bash
# fused push supersteps: parity + cfg3 timing (fused vs the gather/activate pair)
T=${1:-push}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q -p no:cacheprovider -k "sssp or widest or runtime or random or hubs or reduced or custom or cfg3" > gpurun_out/push_tests_$T.log 2>&1
tail -5 gpurun_out/push_tests_$T.log
timeout 600 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/bench_${T}_cfg3.json 2> gpurun_out/bench_${T}_cfg3.err
GR_PUSH_FUSED=0 timeout 600 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/bench_${T}_cfg3_nofuse.json 2> /dev/null
timeout 600 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --loop device > gpurun_out/bench_${T}_cfg3_graph.json 2> /dev/null
for f in gpurun_out/bench_${T}_cfg3*.json; do echo $f; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['value'], d.get('phase_ms_per_step'))"; done
tail -3 gpurun_out/bench_${T}_cfg3.err
