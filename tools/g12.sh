mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_alg2.py tests/test_gpu_n3.py tests/test_gpu_modeg.py -q -x > gpurun_out/pytest_part.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_part.log
L=paper_conf_middleware_bhasisjgpkd24_b200
vb() { timeout 300 python tools/variant_bench.py $L/$1 $2 $3 2>&1 | tail -1 | tee -a gpurun_out/ab12.log; }
vb libprotean_base.so 4096 120; vb libprotean.so 4096 120; vb libprotean_base.so 4096 120; vb libprotean.so 4096 120
PHASE_LIB=libprotean_phase.so timeout 300 python tools/phase_timing.py 444 60 > gpurun_out/phase_new.log 2>&1; cat gpurun_out/phase_new.log
timeout 600 compute-sanitizer --tool racecheck --print-limit 10 python tools/sanitize_run.py c1 > gpurun_out/rc_c1.log 2>&1; tail -2 gpurun_out/rc_c1.log
