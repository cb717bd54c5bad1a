mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --csv -k regex:score_kernel -c 5 python bench.py --path c1 > gpurun_out/ncu_c1.log 2>&1; grep -i "score_kernel" gpurun_out/ncu_c1.log | head -5
timeout 900 python bench.py --path sweep --replicas 4096 --cpu-sample 16 > gpurun_out/bench_sweep.log 2>&1; tail -1 gpurun_out/bench_sweep.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps(d['oracle_gap'])); print(d['value'], d['roofline'])"
