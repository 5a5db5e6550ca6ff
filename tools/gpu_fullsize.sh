#!/bin/bash
# full-size parity tests + default bench line (clock sampler check)
T=${1:-fs}
mkdir -p gpurun_out
python bench.py > gpurun_out/bench_${T}_cfg2.json 2> gpurun_out/bench_${T}_cfg2.err
timeout 1500 python -m pytest tests/test_gpu_fullsize.py -x -q -p no:cacheprovider --durations=0 > gpurun_out/fullsize_$T.log 2>&1
tail -15 gpurun_out/fullsize_$T.log; cat gpurun_out/bench_${T}_cfg2.json
