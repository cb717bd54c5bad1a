mkdir -p gpurun_out
D=paper_conf_middleware_bhasisjgpkd24_b200
for rep in 1 2; do
  timeout 300 python tools/variant_bench.py $D/libprotean.so 4096 120 2>&1 | tail -1
  PROTEAN_WINDOW_SMEM=0 timeout 300 python tools/variant_bench.py $D/libprotean.so 4096 120 2>&1 | tail -1
  PROTEAN_WINDOW_SMEM=0 timeout 300 python tools/variant_bench.py $D/libprotean_m4.so 4096 120 2>&1 | tail -1
  PROTEAN_WINDOW_SMEM=0 timeout 300 python tools/variant_bench.py $D/libprotean_w7.so 4096 120 2>&1 | tail -1
done
