mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "delta or random or reduced or dense or hubs" 2>&1 | tail -2
for v in 1 0; do
  GR_DENSE_SEG=$v timeout 600 python bench.py --config 2 --algo pagerank_delta --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/dsq_f2_$v.json 2>/dev/null
  GR_DENSE_SEG=$v timeout 600 python bench.py --config 1 --algo sssp --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/dsq_c1sssp_$v.json 2>/dev/null
  GR_DENSE_SEG=$v timeout 600 python bench.py --config 4 --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/dsq_cfg4_$v.json 2>/dev/null
  GR_DENSE_SEG=$v timeout 600 python bench.py --config 2 --algo cc --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/dsq_c2cc_$v.json 2>/dev/null
done
for f in gpurun_out/dsq_*.json; do python -c "import json; d=json.load(open('$f')); print('$f', d['ms_per_step'], d['value'], d.get('phase_ms_per_step'))"; done
