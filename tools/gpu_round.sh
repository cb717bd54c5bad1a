#!/bin/bash
# Round check on one B200: build, GPU tests, smoke, bench line, ncu launch list + full capture.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke.log
bash tools/gpu_measure.sh
python bench.py --policy alg2 > gpurun_out/bench_alg2.log 2>&1; tail -1 gpurun_out/bench_alg2.log | cut -c1-200
python bench.py --path sweep --cpu-sample 16 > gpurun_out/bench_sweep.log 2>&1; tail -1 gpurun_out/bench_sweep.log | cut -c1-200
ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -c 1 -o gpurun_out/sweep_full -f python tools/sweep_run.py 512 > gpurun_out/ncu_sweep.log 2>&1
python bench.py --cold-start-us 5000000 > gpurun_out/bench_n3.log 2>&1; tail -1 gpurun_out/bench_n3.log | cut -c1-200
