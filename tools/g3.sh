mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
bash tools/build_phase_variant.sh > gpurun_out/build_phase.log 2>&1
bash tools/build_variant.sh racecheck -DPROTEAN_ACCT_BARRIER=1 > gpurun_out/build_rc.log 2>&1
timeout 600 python -m pytest tests/test_gpu_mig_tables.py tests/test_gpu_edges.py -q > gpurun_out/pytest_mig.log 2>&1; tail -3 gpurun_out/pytest_mig.log
timeout 300 python tools/phase_timing.py 444 60 > gpurun_out/phase.log 2>&1; cat gpurun_out/phase.log
for w in c1 c2 c2many; do PROTEAN_LIB=libprotean_racecheck.so timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_run.py $w > gpurun_out/sanitize_racecheck_barrier_$w.log 2>&1; tail -2 gpurun_out/sanitize_racecheck_barrier_$w.log; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:replay_kernel -c 1 -o gpurun_out/replay_full -f python tools/profile_run.py --replicas 444 --seconds 60 --repeat 1 > gpurun_out/ncu_full.log 2>&1; echo "ncu rc=$?"
