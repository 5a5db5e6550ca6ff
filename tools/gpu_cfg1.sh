# cfg1 (BFS, R-MAT s16, 10 MB: L2-flushed timing) across loops / directions / CTAs per SM
mkdir -p gpurun_out
one() { # tag, env..., args...
  t=$1; shift
  env "$@" > /dev/null
}
run() {
  tag=$1; shift
  timeout 300 env $ENVV python bench.py --config 1 --steps 10 --warmup 3 --no-cpu --e2e-steps 0 "$@" > gpurun_out/c1_$tag.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/c1_$tag.json')); print('$tag', d['ms_per_step'], d['value'], d['phase_ms_per_step'], d['config']['pull_supersteps'], d['gpu_launches'])"
}
ENVV= run default
ENVV= run push --direction push
ENVV= run pull --direction pull
ENVV= run device --loop device
ENVV= run host --loop host
ENVV=GR_PERSIST_CTAS_PER_SM=1 run cta1
ENVV=GR_PERSIST_CTAS_PER_SM=2 run cta2
timeout 300 python bench.py --config 1 --e2e-steps 3 > gpurun_out/c1_full.json 2> gpurun_out/c1_full.err
cat gpurun_out/c1_full.json
