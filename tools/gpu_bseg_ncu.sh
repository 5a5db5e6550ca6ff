#!/bin/bash
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum,lts__t_sectors_op_red.sum,l1tex__m_l1tex2xbar_req_cycles_active.avg.pct_of_peak_sustained_elapsed,lts__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active
for k in seg bseg; do
GR_PR_KERNEL=$k timeout 900 ncu --metrics $M --clock-control none -k regex:"k_pr_b?seg_loop" -c 1 --csv python bench.py --config 5 --scale 26 --mode resident --steps 1 --warmup 1 --no-cpu --e2e-steps 0 > gpurun_out/ncu_s26_$k.csv 2> gpurun_out/ncu_s26_$k.err
done
