#!/bin/bash
# ncu A/B of two libprotean builds on the reduced C5 shape: usage bash tools/ncu_ab.sh A.so B.so
mkdir -p gpurun_out
for L in "$@"; do
  n=$(basename $L .so)
  ncu --set full --clock-control none --import-source on -k regex:replay_kernel -c 1 -o gpurun_out/ab_$n -f python tools/variant_bench.py $L 444 60 > /dev/null 2>&1
done
ls gpurun_out/ab_*
