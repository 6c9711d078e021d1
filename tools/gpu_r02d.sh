set -x
T=r02d
mkdir -p gpurun_out/$T
timeout 300 python tools/probe_outputs.py 2 > gpurun_out/$T/probe_c2.log 2>&1; cat gpurun_out/$T/probe_c2.log | grep graph
timeout 600 ncu --set full --clock-control none --import-source on -k "regex:k_fused_small" -s 2 -c 1 \
  -o gpurun_out/$T/c2_small python bench.py --workload 2 --steps 1 --warmup 3 --e2e-steps 0 --cpu-seconds 0 \
  > gpurun_out/$T/c2_small.log 2>&1; echo ncu rc=$?
timeout 900 python tools/debug_sharded_case.py > gpurun_out/$T/dbg.log 2>&1; grep -v Warn gpurun_out/$T/dbg.log | tail -6
