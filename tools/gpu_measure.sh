#!/bin/bash
# Round measurement: full bench line, ncu launch list of the bench command, one ncu --set full
# capture of replay_kernel on a reduced C5 shape.  Outputs under gpurun_out/.
mkdir -p gpurun_out
python bench.py > gpurun_out/bench_full.log 2>&1
tail -1 gpurun_out/bench_full.log
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 2 --warmup 1 --cpu-sample 0 --e2e-replicas 0 > gpurun_out/bench_ncu.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:replay_kernel -c 1 -o gpurun_out/replay_full -f \
  python tools/profile_run.py --replicas 444 --seconds 60 --repeat 1 > gpurun_out/ncu1.log 2>&1
ls gpurun_out
