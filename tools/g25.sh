mkdir -p gpurun_out
PHASE_MIX=b8 PHASE_N=64 timeout 600 python tools/phase_timing.py 1 600 > gpurun_out/phase_c4.log 2>&1; cat gpurun_out/phase_c4.log
PHASE_MIX=b PHASE_N=8 timeout 600 python tools/phase_timing.py 1 600 > gpurun_out/phase_c2.log 2>&1; cat gpurun_out/phase_c2.log
