T=r02z6
mkdir -p gpurun_out/$T
timeout 300 python tools/probe_online.py 262144 4 fused timing > gpurun_out/$T/fused_timing.log 2>&1; tail -8 gpurun_out/$T/fused_timing.log
timeout 300 python tools/probe_online.py 262144 4 append_hash timing > gpurun_out/$T/ah_timing.log 2>&1; tail -8 gpurun_out/$T/ah_timing.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/$T/fused_launches.csv python tools/probe_online.py 262144 2 fused > gpurun_out/$T/fused_ncu.log 2>&1
python tools/ncu_launch_table.py gpurun_out/$T/fused_launches.csv 2>/dev/null | head -40
