mkdir -p gpurun_out
for c in 1 3 4; do
  for k in 2 3 4; do
    GR_PERSIST_CTAS_PER_SM=$k timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/ctas_${c}_$k.json 2>/dev/null
    python -c "import json; d=json.load(open('gpurun_out/ctas_${c}_$k.json')); print('cfg$c ctas/SM=$k', d['ms_per_step'], d['value'])"
  done
done
