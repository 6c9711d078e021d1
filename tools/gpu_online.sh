T=r02z4
mkdir -p gpurun_out/$T
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider -k "online" > gpurun_out/$T/tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/$T/tests.log
timeout 600 python bench.py --workload 2 --online 1,64,4096,65536,262144 --online-max-windows 2000 --check > gpurun_out/$T/c2_online.json 2> gpurun_out/$T/c2_online.err; echo "bench rc=$?"
python -c "
import json
d=json.load(open('gpurun_out/$T/c2_online.json')); print('batch', d['batch_ms'])
for w in d['windows']: print(w)"
tail -5 gpurun_out/$T/c2_online.err
