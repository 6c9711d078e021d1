set -x
T=r02f
mkdir -p gpurun_out/$T
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,sm__warps_active.avg.pct_of_peak_sustained_active --clock-control none -c 60 --csv \
  --log-file gpurun_out/$T/c2_launches.csv python bench.py --workload 2 --steps 1 --warmup 3 --e2e-steps 0 --cpu-seconds 0 \
  > gpurun_out/$T/c2_launch_bench.log 2>&1
timeout 600 python tools/probe_online.py 65536 8 > gpurun_out/$T/online_65536.log 2>&1
timeout 600 python tools/probe_online.py 4096 64 > gpurun_out/$T/online_4096.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv \
  --log-file gpurun_out/$T/online_launches.csv python tools/probe_online.py 65536 4 > gpurun_out/$T/online_ncu.log 2>&1
cat gpurun_out/$T/online_65536.log gpurun_out/$T/online_4096.log
