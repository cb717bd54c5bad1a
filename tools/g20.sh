mkdir -p gpurun_out
D=paper_conf_middleware_bhasisjgpkd24_b200
for rep in 1 2; do
  for v in mw mwm2 mwk8 mwk6; do
    timeout 300 python tools/variant_bench.py $D/libprotean_$v.so 4096 120 2>&1 | tail -1
  done
done
