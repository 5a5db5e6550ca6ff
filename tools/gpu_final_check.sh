mkdir -p gpurun_out
timeout 1500 python -m pytest tests -x -q -m gpu -p no:cacheprovider 2>&1 | tail -3
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
for c in 1 3 4; do
  timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --e2e-steps 1 > gpurun_out/fin_cfg$c.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/fin_cfg$c.json')); print('cfg$c', d['ms_per_step'], d['value'], d['e2e']['value'])"
done
timeout 600 python bench.py --config 2 --algo pagerank_delta --steps 3 --warmup 3 --e2e-steps 1 > gpurun_out/fin_f2.json 2>/dev/null
timeout 600 python bench.py --config 1 --algo sssp --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/fin_c1sssp.json 2>/dev/null
for f in fin_f2 fin_c1sssp; do python -c "import json; d=json.load(open('gpurun_out/$f.json')); print('$f', d['ms_per_step'], d['value'])"; done
