L=paper_conf_middleware_bhasisjgpkd24_b200
for i in 1 2; do
for v in libprotean libprotean_prev; do python tools/variant_bench.py $L/$v.so 4096 120; done
done
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -2
