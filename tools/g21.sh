mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_fullsize.py tests/test_gpu_alg2.py tests/test_gpu_n3.py tests/test_gpu_modeg.py -q -x > gpurun_out/pytest_part.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_part.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:replay_kernel -c 1 -o gpurun_out/replay_mw -f \
    python tools/profile_run.py --replicas 444 --seconds 60 --repeat 1 > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?"
