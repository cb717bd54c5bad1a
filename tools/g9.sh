mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_validation.py -q -x > gpurun_out/pytest_part.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_part.log
timeout 600 python bench.py --path c1 > gpurun_out/bench_c1.log 2>&1; tail -1 gpurun_out/bench_c1.log | cut -c1-600
timeout 300 compute-sanitizer --tool memcheck python tools/sanitize_run.py score > gpurun_out/sanitize_memcheck_score2.log 2>&1; tail -2 gpurun_out/sanitize_memcheck_score2.log
timeout 300 compute-sanitizer --tool racecheck python tools/sanitize_run.py score > gpurun_out/sanitize_racecheck_score2.log 2>&1; tail -2 gpurun_out/sanitize_racecheck_score2.log
