mkdir -p gpurun_out
D=paper_conf_middleware_bhasisjgpkd24_b200
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_dispatch.py tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_edges.py tests/test_gpu_modeg.py tests/test_gpu_validation.py tests/test_gpu_n3.py tests/test_gpu_alg2.py -q -x > gpurun_out/pytest_part.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_part.log
for p in c2 c4; do for lib in libprotean_base.so libprotean.so; do echo "$lib $(PROTEAN_LIB=$lib timeout 300 python bench.py --path $p --steps 5 --warmup 3 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["metric"], d["value"], d["unit"], d["ms_per_step"])')"; done; done
for v in base ""; do timeout 300 python tools/variant_bench.py $D/libprotean${v:+_$v}.so 4096 120 2>&1 | tail -1; done
