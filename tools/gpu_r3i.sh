#!/bin/bash
# 5 CTAs/SM build A/B (cfg4, cfg3, cfg1); ncu of the PageRank loop, TMA vs load path (summarized on the box)
T=${1:-r3i}
mkdir -p gpurun_out
for v in base c5 base c5; do
  if [ $v = c5 ]; then export GR_LIB=variants/libgr_c5.so GR_PERSIST_CTAS_PER_SM=5; else unset GR_LIB GR_PERSIST_CTAS_PER_SM; fi
  for c in 4 3; do
    timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --other-configs 0 > gpurun_out/${T}_cfg${c}_$v.json 2> gpurun_out/${T}_cfg${c}_$v.err
    echo "cfg$c $v $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/${T}_cfg${c}_$v.json)"
  done
done
unset GR_LIB GR_PERSIST_CTAS_PER_SM
for tma in 1 0; do
  GR_PR_TMA=$tma timeout 600 ncu --set full --clock-control none -k regex:k_pr_seg_loop -c 1 -o /tmp/${T}_pr_tma$tma python tools/run_once.py 2 pagerank auto > gpurun_out/${T}_ncu_tma$tma.log 2>&1
  echo "ncu tma$tma rc=$?"
  python tools/summarize_ncu.py full /tmp/${T}_pr_tma$tma.ncu-rep gpurun_out/${T}_pr_tma$tma.md
  ncu -i /tmp/${T}_pr_tma$tma.ncu-rep --page raw --csv > gpurun_out/${T}_pr_tma${tma}_raw.csv 2>/dev/null
done
ls -la gpurun_out | grep $T
