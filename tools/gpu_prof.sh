#!/bin/bash
# Phase timing (debug build) + one ncu --set full capture of replay_kernel on a reduced C5 shape.
mkdir -p gpurun_out
python tools/phase_timing.py 444 60 > gpurun_out/phase.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:replay_kernel -c 1 -o gpurun_out/replay_full -f python tools/profile_run.py --replicas 444 --seconds 60 --repeat 1 > gpurun_out/ncu1.log 2>&1
cat gpurun_out/phase.txt
