mkdir -p gpurun_out
D=paper_conf_middleware_bhasisjgpkd24_b200
for rep in 1 2; do
  for v in base a1 a2 r1; do
    L=$D/libprotean${v:+_$v}.so
    timeout 300 python tools/variant_bench.py $L 4096 120 2>&1 | tail -1
  done
done
