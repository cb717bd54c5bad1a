#!/bin/bash
# Other bench lines and compute-sanitizer logs on one B200.  Logs under gpurun_out/.
mkdir -p gpurun_out/sanitizer
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 600 python bench.py --replicas 512 --cpu-sample 0 --e2e-replicas 0 > gpurun_out/bench_512.log 2>&1; echo "512 rc=$?"
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.log 2>&1; echo "ref rc=$?"
for p in c1 c2 c4; do timeout 900 python bench.py --path $p --steps 3 --warmup 1 > gpurun_out/bench_$p.log 2>&1; echo "$p rc=$?"; done
timeout 600 python bench.py --policy alg2 --e2e-replicas 0 --cpu-sample 0 > gpurun_out/bench_alg2.log 2>&1; echo "alg2 rc=$?"
timeout 600 python bench.py --cold-start-us 5000000 --keepalive-epochs 600 --e2e-replicas 0 --cpu-sample 0 > gpurun_out/bench_n3.log 2>&1; echo "n3 rc=$?"
timeout 600 python bench.py --path sweep --cpu-sample 16 > gpurun_out/bench_sweep.log 2>&1; echo "sweep rc=$?"
for t in memcheck racecheck synccheck; do
  for w in lean c1 c2many score sweep; do
    timeout 1200 compute-sanitizer --tool $t --print-limit 50 python tools/sanitize_run.py $w > gpurun_out/sanitizer/${t}_${w}.log 2>&1
    echo "sanitize $t $w rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' gpurun_out/sanitizer/${t}_${w}.log | tail -1)"
  done
done
