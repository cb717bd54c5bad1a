#!/bin/bash
# One GPU round trip: parity tests (-m gpu), smoke, bench line.  Usage: bash tools/gpu_check.sh [pytest -k expr]
mkdir -p gpurun_out
K=${1:-}
if [ -n "$K" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q -k "$K" 2>&1 | tail -25 > gpurun_out/gputests.log
else
  timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -25 > gpurun_out/gputests.log
fi
tail -3 gpurun_out/gputests.log
timeout 300 python bench.py --cpu-sample 0 --e2e-replicas 0 > gpurun_out/bench.log 2>&1
tail -1 gpurun_out/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('ms/step', d['ms_per_step'], 'kernel', r['kernel_ms'], 'prepass', r['prepass_ms'], 'frac', r['frac'], 'value', d['value'])" || tail -5 gpurun_out/bench.log
