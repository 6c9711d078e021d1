#!/bin/bash
# Build tuning variants of libffm.so (same sources, different compile-time knobs) into
# build/variants/<name>/libffm.so; select one with bench.py --lib <path> / pytest --ffm-lib <path>.
# usage: tools/build_variants.sh name:"-DKNOB=V -DKNOB2=V" ...
set -eu
cd "$(dirname "$0")/.."
C=paper_conf_sc_weltonm19_b200/csrc
for spec in "$@"; do
  name=${spec%%:*}; defs=${spec#*:}
  mkdir -p build/variants/$name
  /usr/local/cuda/bin/nvcc -shared -Xcompiler -fPIC,-fopenmp -O3 -lineinfo -std=c++17 -gencode arch=compute_100a,code=sm_100a \
    $defs $C/kernels.cu $C/shard.cu $C/online.cu $C/comm.cu $C/ffm_api.cu $C/shard_plan.cpp -ldl -lgomp -o build/variants/$name/libffm.so &
done
wait
ls -la build/variants/*/libffm.so
