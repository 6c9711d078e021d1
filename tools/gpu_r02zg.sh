T=r02zg
mkdir -p gpurun_out/$T
timeout 1200 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/$T/tests.log
bash tools/gpu_ab.sh $T "2 5 3" "-" "prev" 2
timeout 600 python bench.py --workload 2 --online 1,64,4096,65536,262144,524288,1000000 --check > gpurun_out/$T/c2_online.json 2> gpurun_out/$T/c2_online.err; echo "online rc=$?"
python -c "
import json
d=json.load(open('gpurun_out/$T/c2_online.json')); print('batch', d['batch_ms'])
for w in d['windows']: print(w['mode'], w['window'], w['windows'], 'step', w['step_ms_median'], 'p90', w['step_ms_p90'], 'steps_only', w['steps_only_gbs'], w.get('parity'))"
