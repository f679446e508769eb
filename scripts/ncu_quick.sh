#!/bin/bash
# quick ncu counters for the warp-bin kernel of one nu-LPA run (2 sweeps)
# usage: bash scripts/ncu_quick.sh <kernel-regex> <out-name> [env...]
K=${1:-k_warp}; O=${2:-quick}
ncu --clock-control none -k regex:$K -c 2 --csv --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,launch__registers_per_thread,smsp__average_warp_latency_issue_stalled_long_scoreboard,smsp__warp_issue_stalled_long_scoreboard_per_warp_active.pct,smsp__warp_issue_stalled_mio_throttle_per_warp_active.pct,smsp__warp_issue_stalled_lg_throttle_per_warp_active.pct,smsp__warp_issue_stalled_short_scoreboard_per_warp_active.pct,smsp__warp_issue_stalled_no_instruction_per_warp_active.pct,smsp__warp_issue_stalled_wait_per_warp_active.pct,smsp__warp_issue_stalled_math_pipe_throttle_per_warp_active.pct,smsp__warp_issue_stalled_barrier_per_warp_active.pct,smsp__warp_issue_stalled_membar_per_warp_active.pct,smsp__warp_issue_stalled_branch_resolving_per_warp_active.pct,smsp__warp_issue_stalled_dispatch_stall_per_warp_active.pct \
  python scripts/profile_run.py --runs 1 > gpurun_out/$O.csv 2>&1
python scripts/ncu_table.py gpurun_out/$O.csv
