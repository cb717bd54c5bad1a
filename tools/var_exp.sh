L=paper_conf_middleware_bhasisjgpkd24_b200
python tools/variant_bench.py $L/libprotean.so
PROTEAN_WINDOW_SMEM=0 python tools/variant_bench.py $L/libprotean.so
python tools/variant_bench.py $L/libprotean_minb4.so
PROTEAN_WINDOW_SMEM=0 python tools/variant_bench.py $L/libprotean_minb4.so
