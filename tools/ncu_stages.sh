#!/bin/bash
# ncu metrics of the production kernel at TMA ring depth 4 vs 5 (explains profiles/ab_stages_r01.txt)
set -e
mkdir -p gpurun_out build
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__warps_active.avg.pct_of_peak_sustained_active,launch__grid_size,launch__shared_mem_per_block_dynamic,launch__occupancy_limit_shared_mem,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,lts__t_sector_hit_rate.pct,smsp__average_warp_latency_issue_stalled_long_scoreboard.ratio,smsp__average_warp_latency_issue_stalled_barrier.ratio,l1tex__t_sector_hit_rate.pct
for s in 4 5; do
  python -c "
from paper_conf_icpp_tiankexc16_b200 import build as b
b.build(force=True, extra=['-DSAFARA_TY=12','-DSAFARA_STAGES=$s','-DSAFARA_RCP=2'], out='build/libsafara_s$s.so')" > /dev/null
  SAFARA_LIB=build/libsafara_s$s.so ncu --metrics $M --clock-control none -k regex:rhs_kernel -c 3 \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --soak-s 0 --e2e-steps 0 > gpurun_out/ncu_stages_s$s.txt 2>&1 || true
done
