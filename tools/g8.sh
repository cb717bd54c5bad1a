mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench_full.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench_full.log | cut -c1-300
timeout 600 python bench.py --replicas 512 --cpu-sample 0 --e2e-replicas 0 > gpurun_out/bench_512.log 2>&1; tail -1 gpurun_out/bench_512.log | cut -c1-300
timeout 600 python tools/ncu_capture.py run --replicas 444 --seconds 60 > gpurun_out/ncu_capture.log 2>&1; echo "ncu_capture rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 2 --warmup 1 --cpu-sample 0 --e2e-replicas 0 > gpurun_out/bench_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:replay_kernel -c 1 -o gpurun_out/replay_full -f \
    python tools/profile_run.py --replicas 444 --seconds 60 --repeat 1 > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?"
for p in c1 c2 c4; do timeout 900 python bench.py --path $p --steps 3 --warmup 1 > gpurun_out/bench_$p.log 2>&1; echo "$p rc=$?"; done
timeout 600 python bench.py --policy alg2 --e2e-replicas 0 > gpurun_out/bench_alg2.log 2>&1; tail -1 gpurun_out/bench_alg2.log | cut -c1-200
timeout 600 python bench.py --path sweep --cpu-sample 16 > gpurun_out/bench_sweep.log 2>&1; tail -1 gpurun_out/bench_sweep.log | cut -c1-200
timeout 600 python bench.py --cold-start-us 5000000 --e2e-replicas 0 --cpu-sample 8 > gpurun_out/bench_n3.log 2>&1; tail -1 gpurun_out/bench_n3.log | cut -c1-200
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.log 2>&1; tail -1 gpurun_out/bench_ref.log | cut -c1-200
