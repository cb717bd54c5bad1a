#!/bin/bash
# Key ncu counters of replay_kernel for policy 0 and policy 2 on a reduced C5 shape.
mkdir -p gpurun_out
M=gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__thread_inst_executed_per_inst_executed.ratio,sm__cycles_elapsed.avg,smsp__average_warp_latency_issue_stalled_barrier,smsp__warp_issue_stalled_barrier_per_warp_active.pct,smsp__warp_issue_stalled_no_instruction_per_warp_active.pct,smsp__warp_issue_stalled_wait_per_warp_active.pct,smsp__warp_issue_stalled_short_scoreboard_per_warp_active.pct,smsp__warp_issue_stalled_long_scoreboard_per_warp_active.pct,smsp__warp_issue_stalled_sleeping_per_warp_active.pct,smsp__warp_issue_stalled_membar_per_warp_active.pct,smsp__warp_issue_stalled_branch_resolving_per_warp_active.pct,smsp__warp_issue_stalled_math_pipe_throttle_per_warp_active.pct,smsp__warp_issue_stalled_lg_throttle_per_warp_active.pct,smsp__warp_issue_stalled_mio_throttle_per_warp_active.pct,smsp__warp_issue_stalled_dispatch_stall_per_warp_active.pct
for pol in 0 2; do
  ncu --metrics $M --clock-control none -k regex:replay_kernel -c 1 --csv python tools/policy_time.py 444:120:$pol 2>/dev/null | grep replay_kernel | awk -F'","' '{print $(NF-2)": "$NF}' | sed 's/"//g' > gpurun_out/ncu_policy$pol.txt
  echo "== policy $pol"; cat gpurun_out/ncu_policy$pol.txt
done
