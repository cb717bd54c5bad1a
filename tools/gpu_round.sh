#!/bin/bash
# Round-2 check on one B200: build, GPU tests, smoke, bench lines, ncu metrics + full capture,
# compute-sanitizer logs.  Everything lands in gpurun_out/ (copy what is judged into profiles/).
mkdir -p gpurun_out
free -g > gpurun_out/host_mem.txt; nproc >> gpurun_out/host_mem.txt; lscpu | head -20 >> gpurun_out/host_mem.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
STAGE=${STAGE:-all}
if [[ $STAGE == all || $STAGE == tests ]]; then
  timeout 2400 python -m pytest tests -m gpu -q -x ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke.log
fi
if [[ $STAGE == all || $STAGE == bench ]]; then
  timeout 900 python bench.py > gpurun_out/bench_full.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench_full.log | cut -c1-300
  timeout 600 python tools/ncu_capture.py run --replicas 444 --seconds 60 > gpurun_out/ncu_capture.log 2>&1; echo "ncu_capture rc=$?"
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 2 --warmup 1 --cpu-sample 0 --e2e-replicas 0 > gpurun_out/bench_ncu.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:replay_kernel -c 1 -o gpurun_out/replay_full -f \
    python tools/profile_run.py --replicas 444 --seconds 60 --repeat 1 > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?"
fi
if [[ $STAGE == all || $STAGE == paths ]]; then
  for p in c1 c2 c4; do timeout 900 python bench.py --path $p --steps 3 --warmup 1 > gpurun_out/bench_$p.log 2>&1; echo "$p rc=$?"; tail -1 gpurun_out/bench_$p.log | cut -c1-200; done
  timeout 600 python bench.py --policy alg2 --e2e-replicas 0 > gpurun_out/bench_alg2.log 2>&1; tail -1 gpurun_out/bench_alg2.log | cut -c1-200
  timeout 600 python bench.py --path sweep --cpu-sample 16 > gpurun_out/bench_sweep.log 2>&1; tail -1 gpurun_out/bench_sweep.log | cut -c1-200
fi
if [[ $STAGE == all || $STAGE == sanitize ]]; then
  for t in racecheck synccheck memcheck; do
    for w in c1 score sweep c2 c2many; do
      timeout 1200 compute-sanitizer --tool $t --print-limit 50 python tools/sanitize_run.py $w > gpurun_out/sanitize_${t}_${w}.log 2>&1
      echo "sanitize $t $w rc=$?"; tail -2 gpurun_out/sanitize_${t}_${w}.log
    done
  done
fi
ls gpurun_out
