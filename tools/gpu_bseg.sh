#!/bin/bash
# source-blocked PageRank (f3): parity + s26 resident sweep of block size / policy
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "source_blocked" 2>&1 | tail -2
b() { timeout 900 python bench.py --config 5 --scale 26 --mode resident --steps 2 --warmup 2 --no-cpu --e2e-steps 0 > gpurun_out/b_$1.json 2>gpurun_out/b_$1.err; python -c "import json;d=json.load(open('gpurun_out/b_$1.json'));print('$1',d['value'],d['ms_per_step'],d['roofline']['kernel'],d['roofline']['avg_launch_us'],d['roofline']['frac'])" || tail -3 gpurun_out/b_$1.err; }
for mb in 40 24 64; do GR_PR_BLOCK_MB=$mb b s26_bseg_mb$mb; done
GR_PR_BLOCK_POLICY=0 b s26_bseg_nopol
