#!/bin/bash
# Round evidence on one B200: the bench line, per-kernel ncu metrics, the launch list of the bench
# command, and one ncu --set full capture of the dominant kernel.  Logs under gpurun_out/.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1200 python bench.py > gpurun_out/bench_full.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench_full.log | cut -c1-300
timeout 900 python tools/ncu_capture.py run --replicas 4096 --seconds 60 > gpurun_out/ncu_capture.log 2>&1; echo "ncu_capture rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 2 --warmup 1 --cpu-sample 0 --e2e-replicas 0 > gpurun_out/bench_ncu.log 2>&1; echo "launches rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"cand_kernel|chain_kernel|acct_kernel" -c 3 \
  -o gpurun_out/lean_full -f python tools/profile_run.py --replicas 4096 --seconds 60 --repeat 1 > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?"
ls gpurun_out
