#!/bin/bash
# A/B of the working-tree libprotean.so against libprotean_base.so (the previous commit) on the
# C5 shape (4096 replicas x S s), then the GPU tests.  Outputs under gpurun_out/.
mkdir -p gpurun_out
S=${S:-120}
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
for rep in 1 2; do
  for lib in libprotean_base.so libprotean.so; do
    timeout 300 python tools/variant_bench.py paper_conf_middleware_bhasisjgpkd24_b200/$lib 4096 $S 2>&1 | tail -1 | tee -a gpurun_out/ab.log
  done
done
if [[ -n "$TESTS" ]]; then
  timeout 2400 python -m pytest tests -m gpu -q $TESTS > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_gpu.log
fi
