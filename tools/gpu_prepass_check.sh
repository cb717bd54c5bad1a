#!/bin/bash
# GPU tests, a prepass/partition ncu timing pass and a kernel-only bench line.
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gputests.log 2>&1; tail -1 gpurun_out/gputests.log
ncu --metrics gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum --clock-control none -k "regex:part_|prepass" -c 4 --csv --log-file gpurun_out/prepass.csv python tools/profile_run.py --replicas 1024 --seconds 600 --repeat 1 > /dev/null 2>&1
grep prepass gpurun_out/prepass.csv | cut -c1-40,200-
timeout 300 python bench.py --cpu-sample 0 --e2e-replicas 0 > gpurun_out/bench.log 2>&1; tail -1 gpurun_out/bench.log | cut -c1-200
