mkdir -p gpurun_out
D=paper_conf_middleware_bhasisjgpkd24_b200
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for rep in 1 2; do
  for v in ovl0 ""; do
    L=$D/libprotean${v:+_$v}.so
    timeout 300 python tools/variant_bench.py $L 4096 120 2>&1 | tail -1
  done
done
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_fullsize.py tests/test_gpu_n3.py tests/test_gpu_modeg.py tests/test_gpu_validation.py -q -x > gpurun_out/pytest_part.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_part.log
