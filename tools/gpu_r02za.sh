T=r02za
mkdir -p gpurun_out/$T
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider -k "online or smoke or golden or configs_reduced" > gpurun_out/$T/tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/$T/tests.log
timeout 600 python bench.py --workload 2 --online 1,64,4096,65536,262144 --online-max-windows 2000 --check > gpurun_out/$T/c2_online.json 2> gpurun_out/$T/c2_online.err; echo "online rc=$?"
python -c "
import json
d=json.load(open('gpurun_out/$T/c2_online.json')); print('batch', d['batch_ms'])
for w in d['windows']: print(w['mode'], w['window'], w['windows'], 'step', w['step_ms_median'], 'append', w['append_ms_median'], 'steps_only', w['steps_only_gbs'], 'streamed', w['streamed_gbs'], w.get('parity'))"
tail -3 gpurun_out/$T/c2_online.err
