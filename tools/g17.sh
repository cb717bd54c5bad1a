mkdir -p gpurun_out
for rep in 1 2; do
for lib in libprotean_base.so libprotean_n64.so libprotean_n32.so; do
  for p in c4; do
    echo "$lib $p $(PROTEAN_LIB=$lib timeout 300 python bench.py --path $p --steps 5 --warmup 3 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["unit"], d["ms_per_step"])')"
  done
done
done
PROTEAN_LIB=libprotean_n64.so timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_modeg.py -q -x > gpurun_out/pytest_n64.log 2>&1; echo "pytest n64 rc=$?"; tail -3 gpurun_out/pytest_n64.log
