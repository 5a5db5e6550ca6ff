#!/bin/bash
# ncu of the fused push phase vs the gather/activate pair on cfg3 (host loop, mid-run supersteps)
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none -k regex:k_push_expand --launch-skip 5000 -c 2 -o gpurun_out/push_fused -f python bench.py --config 3 --steps 1 --warmup 0 --no-cpu --e2e-steps 0 --loop host > gpurun_out/ncu_push.log 2>&1
GR_PUSH_FUSED=0 timeout 900 ncu --set full --clock-control none -k regex:"k_gather_apply|k_activate" --launch-skip 10000 -c 4 -o gpurun_out/push_nofuse -f python bench.py --config 3 --steps 1 --warmup 0 --no-cpu --e2e-steps 0 --loop host >> gpurun_out/ncu_push.log 2>&1
tail -5 gpurun_out/ncu_push.log; ls -la gpurun_out/*.ncu-rep
