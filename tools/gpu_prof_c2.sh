# ncu of the config 2 step: launch list + full set (source-level) of the small-payload pass
set -x
T=${1:-r02b}
mkdir -p gpurun_out/$T
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/$T/c2_launches.csv python bench.py --workload 2 --steps 2 --warmup 3 --e2e-steps 0 --cpu-seconds 0 \
  > gpurun_out/$T/c2_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on \
  -k "regex:k_fused_small|k_group_insert|k_leader0|k_label_hist" -s 8 -c 4 \
  -o gpurun_out/$T/c2_prof python bench.py --workload 2 --steps 1 --warmup 3 --e2e-steps 0 --cpu-seconds 0 \
  > gpurun_out/$T/c2_full_bench.log 2>&1
timeout 600 python bench.py --workload 2 --steps 20 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c2_bench.json 2> gpurun_out/$T/c2_bench.err
tail -c 1500 gpurun_out/$T/c2_bench.json
ls -la gpurun_out/$T
