#!/bin/bash
# Copy one tools/gpu_round.sh run (gpurun_out/) into profiles/<tag>_*.
T=$1
python tools/make_profiles.py $T > /dev/null 2>&1
for k in alg2 sweep n3; do tail -1 gpurun_out/bench_$k.log | python -m json.tool > profiles/${T}_${k}_bench_line.json; done
(echo "# ncu --set full, sweep_kernel, tools/sweep_run.py 512 (config-5-shaped GPU-epochs, 4096 units)"
 ncu -i gpurun_out/sweep_full.ncu-rep --page details --csv 2>/dev/null | python -c "
import csv,sys
want=['Duration','Executed Ipc Active','Issue Slots Busy','Achieved Occupancy','Theoretical Occupancy','Registers Per Thread','Avg. Active Threads Per Warp','Warp Cycles Per Issued Instruction','Eligible Warps Per Scheduler','Compute (SM) Throughput','Block Limit Registers','Branch Efficiency','DRAM Throughput','Memory Throughput']
seen=set()
for r in csv.reader(sys.stdin):
    if len(r)>14 and r[12] in want and r[12] not in seen: seen.add(r[12]); print(f'{r[12]:40s} {r[14]:>14s} {r[13]}')
"
 echo "top source lines (stall samples %, instructions %):"
 python - <<'PY'
import sys; sys.path.insert(0,'tools')
import ncu_lines
rows = ncu_lines.lines('gpurun_out/sweep_full.ncu-rep')
tot = sum(r[1] for r in rows); ts=sum(r[0] for r in rows)
for r in sorted(rows, key=lambda r: -r[0])[:16]:
    print(f"  {100*r[0]/ts:4.1f}% {100*r[1]/tot:5.1f}%i {r[2]}:{r[3]} {r[4][:90]}")
PY
) > profiles/${T}_sweep_kernel_ncu_full.txt
python -c "
import json
for f in ['bench_line','alg2_bench_line','sweep_bench_line','n3_bench_line']:
    d=json.load(open('profiles/$T'+'_'+f+'.json')); print(f, round(d['ms_per_step'],1), '%.3g'%d['value'], round(d['roofline']['frac'],4), d['roofline'].get('kernel_ms'), d['clocks'])
"
