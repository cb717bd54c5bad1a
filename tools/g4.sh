mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
L=paper_conf_middleware_bhasisjgpkd24_b200
vb() { timeout 300 python tools/variant_bench.py $L/$1 $2 $3 2>&1 | tail -1 | tee -a gpurun_out/ab4.log; }
vb libprotean_base.so 4096 120; vb libprotean.so 4096 120; vb libprotean_base.so 4096 120; vb libprotean.so 4096 120
vb libprotean.so 512 600
PROTEAN_WINDOW_SMEM=0 vb libprotean_w6.so 512 600
PROTEAN_WINDOW_SMEM=0 vb libprotean.so 512 600
PROTEAN_WINDOW_SMEM=0 vb libprotean_w6.so 4096 120
PROTEAN_WINDOW_SMEM=0 vb libprotean.so 4096 120
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_gpu.log
