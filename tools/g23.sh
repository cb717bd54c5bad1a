mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_validation.py tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_fullsize.py tests/test_gpu_modeg.py tests/test_gpu_modeg_ipc.py tests/test_gpu_form.py -q -x > gpurun_out/pytest_part.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_part.log
for p in c2 c4; do timeout 300 python bench.py --path $p --steps 5 --warmup 3 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["metric"], d["value"], d["unit"], d["ms_per_step"])'; done
