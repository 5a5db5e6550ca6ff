#!/bin/bash
# dense edge-segmented gather: parity + cfg4 CC / cfg2 PageRank-delta with and without (GR_DENSE_SEG=0)
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q -p no:cacheprovider -k "not streamed" > gpurun_out/dseg_tests.log 2>&1
tail -4 gpurun_out/dseg_tests.log
for v in 1 0; do
  GR_DENSE_SEG=$v timeout 600 python bench.py --config 4 --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/dseg_cfg4_$v.json 2>/dev/null
  GR_DENSE_SEG=$v timeout 600 python bench.py --config 2 --algo pagerank_delta --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/dseg_f2_$v.json 2>/dev/null
  GR_DENSE_SEG=$v timeout 600 python bench.py --config 1 --algo sssp --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/dseg_c1sssp_$v.json 2>/dev/null
done
for f in gpurun_out/dseg_*.json; do python -c "import json; d=json.load(open('$f')); print('$f', d['ms_per_step'], d['value'], d['config'].get('iterations'), d['config'].get('pull_supersteps'), d.get('phase_ms_per_step'))"; done
