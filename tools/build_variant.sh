#!/bin/bash
# Build a libprotean variant with extra nvcc defines: tools/build_variant.sh NAME -DX=Y ...
set -e
D=/root/repo/paper_conf_middleware_bhasisjgpkd24_b200
N=$1; shift
nvcc "$@" -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -I/root/repo/include \
  -Xcompiler -fPIC -shared -cudart static -o $D/libprotean_$N.so $D/csrc/api.cu $D/csrc/replay.cu $D/csrc/partition.cu $D/csrc/score.cu $D/csrc/sweep.cu $D/csrc/form.cu $D/csrc/cand.cu $D/csrc/chain.cu
