#!/bin/bash
# quick re-validation: all GPU tests, smoke, default bench line
T=${1:-chk}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -x -q -m gpu -p no:cacheprovider 2>&1 | tail -30 > gpurun_out/gpu_tests_$T.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$T.log 2>&1
python bench.py > gpurun_out/bench_${T}_cfg2.json 2> gpurun_out/bench_${T}_cfg2.err
tail -3 gpurun_out/gpu_tests_$T.log; cat gpurun_out/smoke_$T.log | tail -2; cat gpurun_out/bench_${T}_cfg2.json
