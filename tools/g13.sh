mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_tail_split.py tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x > gpurun_out/pytest_part.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_part.log
L=paper_conf_middleware_bhasisjgpkd24_b200
vb() { timeout 300 python tools/variant_bench.py $L/$1 $2 $3 2>&1 | tail -1 | tee -a gpurun_out/ab13.log; }
vb libprotean.so 4096 120; PROTEAN_NO_TAIL_SPLIT=1 vb libprotean.so 4096 120
vb libprotean.so 512 600; PROTEAN_NO_TAIL_SPLIT=1 vb libprotean.so 512 600
timeout 600 python bench.py --cpu-sample 0 --e2e-replicas 0 > gpurun_out/bench_full.log 2>&1; tail -1 gpurun_out/bench_full.log | cut -c1-250
timeout 600 python bench.py --replicas 512 --cpu-sample 0 --e2e-replicas 0 > gpurun_out/bench_512.log 2>&1; tail -1 gpurun_out/bench_512.log | cut -c1-250
