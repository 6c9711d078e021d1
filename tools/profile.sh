#!/bin/bash
# Run on the GPU box (under gpurun): launch list + ncu --set full of the hot kernels.
# usage: tools/profile.sh <tag> [bench args...]
set -u
TAG=$1; shift
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 800 --csv \
  --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 3 --e2e-steps 0 --cpu-seconds 0 "$@" \
  > gpurun_out/${TAG}_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on \
  -k "regex:k_hash_large|k_fused|k_verify_small|k_hash_small|k_group_insert|k_label_hist|k_leader0|k_hash_combine" -s 8 -c 8 \
  -o gpurun_out/${TAG}_prof python bench.py --steps 1 --warmup 3 --e2e-steps 0 --cpu-seconds 0 "$@" \
  > gpurun_out/${TAG}_full_bench.log 2>&1
echo profile-done
