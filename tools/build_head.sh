#!/bin/bash
# Build the committed HEAD's libprotean into libprotean_base.so (A/B baseline for tools/variant_bench.py).
set -e
R=/root/repo
T=$(mktemp -d)
mkdir -p $T/x/y/csrc $T/x/include
for f in $(git -C $R ls-files paper_conf_middleware_bhasisjgpkd24_b200/csrc); do git -C $R show HEAD:$f > $T/x/y/csrc/$(basename $f); done
for f in $(git -C $R ls-files include); do git -C $R show HEAD:$f > $T/x/include/$(basename $f); done
cd $T/x/y/csrc
nvcc "$@" -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -shared -cudart static \
  -o $R/paper_conf_middleware_bhasisjgpkd24_b200/libprotean_base.so api.cu replay.cu partition.cu score.cu sweep.cu form.cu cand.cu chain.cu
rm -rf $T
