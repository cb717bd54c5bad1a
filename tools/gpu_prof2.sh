#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_validation.py -x -q 2>&1 | tail -3
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/part_launches.csv python tools/profile_run.py --replicas 4096 --seconds 60 --repeat 1 > /dev/null 2>&1
grep -E "part_|prepass|replay_kernel" gpurun_out/part_launches.csv | cut -d, -f5,13- | head -40
