#!/bin/bash
# One build -> GPU tests -> bench iteration on a B200 (gpurun); logs under gpurun_out/.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/pytest_gpu.log | cut -c1-300
for v in ${BENCH_VARIANTS:-1}; do
  PROTEAN_PRECAND=$v timeout 600 python bench.py --steps 5 --warmup 3 --cpu-sample 0 --e2e-replicas 0 > gpurun_out/bench_pre$v.log 2>&1
  echo "precand=$v rc=$?"; tail -1 gpurun_out/bench_pre$v.log | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["ms_per_step"], d["value"], d["roofline"]["kernel_ms"], d["roofline"].get("search_ms"))'
done
