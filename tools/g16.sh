mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_fullsize.py tests/test_gpu_alg2.py tests/test_gpu_n3.py tests/test_gpu_modeg.py -q -x > gpurun_out/pytest_part.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_part.log
for rep in 1 2; do
for lib in libprotean_base.so libprotean.so; do
  for p in c2 c4; do
    echo "$lib $p $(PROTEAN_LIB=$lib timeout 300 python bench.py --path $p --steps 5 --warmup 3 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["unit"], d["ms_per_step"])')"
  done
done
done
PHASE_MIX=b timeout 600 python tools/phase_timing.py 1 600 > gpurun_out/phase_c2.log 2>&1; cat gpurun_out/phase_c2.log
