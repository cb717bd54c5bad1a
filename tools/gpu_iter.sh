#!/bin/bash
# Fast GPU iteration: parity subset, phase timing (debug build), kernel-only bench line.
mkdir -p gpurun_out
timeout 600 python -m pytest ${TESTS:-tests/test_gpu_parity.py} -x -q 2>&1 | tail -15
python tools/phase_timing.py 444 60 2>&1 | tail -14
timeout 300 python bench.py --cpu-sample 0 --e2e-replicas 0 > gpurun_out/bench.log 2>&1
tail -1 gpurun_out/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('ms/step', d['ms_per_step'], 'kernel', r['kernel_ms'], 'prepass', r['prepass_ms'], 'frac', r['frac'], 'value', d['value'])" || tail -5 gpurun_out/bench.log
