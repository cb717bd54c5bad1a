#!/bin/bash
# One ncu --set full capture of replay_kernel on a reduced C5 shape (444 replicas x 60 s).
mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on -k regex:replay_kernel -c 1 -o gpurun_out/replay_full -f python tools/profile_run.py --replicas 444 --seconds 60 --repeat 1 > gpurun_out/ncu1.log 2>&1
tail -2 gpurun_out/ncu1.log
