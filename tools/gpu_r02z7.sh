T=r02z7
mkdir -p gpurun_out/$T
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider -k "online or smoke or golden" > gpurun_out/$T/tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/$T/tests.log
timeout 600 python bench.py --workload 2 --online 1,64,4096,65536,262144 --online-max-windows 2000 --check > gpurun_out/$T/c2_online.json 2> gpurun_out/$T/c2_online.err; echo "online rc=$?"
python -c "
import json
d=json.load(open('gpurun_out/$T/c2_online.json')); print('batch', d['batch_ms'])
for w in d['windows']: print(w['mode'], w['window'], w['windows'], 'step', w['step_ms_median'], 'append', w['append_ms_median'], 'steps_only', w['steps_only_gbs'], 'streamed', w['streamed_gbs'], w.get('parity'))"
timeout 300 python tools/probe_online.py 262144 4 fused timing > gpurun_out/$T/fused_timing.log 2>&1; tail -6 gpurun_out/$T/fused_timing.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/$T/fused_launches.csv python tools/probe_online.py 262144 2 fused > gpurun_out/$T/fused_ncu.log 2>&1
python tools/ncu_launch_table.py gpurun_out/$T/fused_launches.csv 2>/dev/null | head -30
