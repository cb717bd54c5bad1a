#!/bin/bash
# Debug build of libprotean with per-phase clock64 instrumentation (tools/phase_timing.py).
set -e
D=/root/repo/paper_conf_middleware_bhasisjgpkd24_b200
nvcc -DPROTEAN_PHASE_TIMING -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 \
  -Xcompiler -fPIC -shared -cudart static -o $D/libprotean_phase.so $D/csrc/api.cu $D/csrc/replay.cu $D/csrc/partition.cu $D/csrc/score.cu $D/csrc/sweep.cu $D/csrc/form.cu $D/csrc/cand.cu $D/csrc/chain.cu
