T=r02z8
mkdir -p gpurun_out/$T
timeout 1200 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/$T/tests.log
bash tools/gpu_ab.sh $T "2 5" "-" "" 2
timeout 600 python bench.py --workload 2 --online 1,64,4096,65536,262144 --online-max-windows 2000 --check > gpurun_out/$T/c2_online.json 2> gpurun_out/$T/c2_online.err; echo "online rc=$?"
python -c "
import json
d=json.load(open('gpurun_out/$T/c2_online.json')); print('batch', d['batch_ms'])
for w in d['windows']: print(w['mode'], w['window'], w['windows'], 'step', w['step_ms_median'], 'append', w['append_ms_median'], 'steps_only', w['steps_only_gbs'], 'streamed', w['streamed_gbs'], w.get('parity'))"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/$T/c2_launches.csv python bench.py --workload 2 --steps 2 --warmup 3 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c2_ncu.log 2>&1
python tools/ncu_launch_table.py gpurun_out/$T/c2_launches.csv | head -12
