mkdir -p gpurun_out
D=paper_conf_middleware_bhasisjgpkd24_b200
for rep in 1 2; do
  for ps in 1 2 3; do
    PROTEAN_PER_SM=$ps timeout 300 python tools/variant_bench.py $D/libprotean.so 888 120 2>&1 | tail -1
  done
done
