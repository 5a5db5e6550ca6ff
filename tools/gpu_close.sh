mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "random or hubs or reduced or repeated or max_iters or custom or dense" 2>&1 | tail -2
for c in 1 3 4; do
  timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/close_cfg$c.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/close_cfg$c.json')); print('cfg$c', d['ms_per_step'], d['value'])"
done
