#!/bin/bash
# Build libffm.so from a git revision (default HEAD) into build/variants/<name>/ for A/B
# runs against the working tree (bench.py --lib build/variants/<name>/libffm.so).
# usage: tools/build_prev.sh [rev] [name]
set -eu
cd "$(dirname "$0")/.."
REV=${1:-HEAD}; NAME=${2:-prev}
T=$(mktemp -d)
git archive "$REV" paper_conf_sc_weltonm19_b200/csrc include | tar -x -C "$T"
C=$T/paper_conf_sc_weltonm19_b200/csrc
mkdir -p build/variants/$NAME
/usr/local/cuda/bin/nvcc -shared -Xcompiler -fPIC,-fopenmp -O3 -lineinfo -std=c++17 -gencode arch=compute_100a,code=sm_100a \
  $C/kernels.cu $C/shard.cu $C/online.cu $C/comm.cu $C/ffm_api.cu $C/shard_plan.cpp -ldl -lgomp -o build/variants/$NAME/libffm.so
rm -rf "$T"
ls -la build/variants/$NAME/libffm.so
