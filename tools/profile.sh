#!/bin/bash
# Run on the GPU box (under gpurun): launch list + ncu --set full of the hot kernels.
# usage: tools/profile.sh <tag> [bench args...]
set -u
TAG=$1; shift
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 800 --csv \
  --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 3 --e2e-steps 0 --cpu-seconds 0 "$@" \
  > gpurun_out/${TAG}_launch_bench.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on \
  -k "regex:k_fused_fx|k_fused_small|k_prefix_hash|k_hash_large|k_hash_small|k_verify_small|k_group_insert|k_leader0|k_label_hist|k_fx_fill|k_hash_combine" -s 12 -c 12 \
  -o gpurun_out/${TAG}_prof python bench.py --steps 1 --warmup 3 --e2e-steps 0 --cpu-seconds 0 "$@" \
  > gpurun_out/${TAG}_full_bench.log 2>&1
echo profile-done
