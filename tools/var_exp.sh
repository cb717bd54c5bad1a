L=paper_conf_middleware_bhasisjgpkd24_b200
for v in libprotean libprotean_w10m2 libprotean_w12m2 libprotean_w16m2; do python tools/variant_bench.py $L/$v.so 4096 120; done
