set -x
T=r02j
mkdir -p gpurun_out/$T
timeout 900 python -m pytest tests/test_gpu_online.py tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo tests rc=$?; tail -3 gpurun_out/$T/tests.log
timeout 600 python tools/probe_online.py 65536 8 > gpurun_out/$T/online_65536.log 2>&1; cat gpurun_out/$T/online_65536.log
timeout 600 python tools/probe_online.py 4096 64 > gpurun_out/$T/online_4096.log 2>&1; cat gpurun_out/$T/online_4096.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv \
  --log-file gpurun_out/$T/online_launches.csv python tools/probe_online.py 65536 4 > gpurun_out/$T/online_ncu.log 2>&1
timeout 900 python bench.py --workload 2 --online 1,64,4096,65536,262144 --check > gpurun_out/$T/c2_online.json 2> gpurun_out/$T/c2_online.err; echo online rc=$?
python -c "
import json; d=json.load(open('gpurun_out/r02j/c2_online.json')); print(d['batch_ms'], d['batch_gbs']); [print(w) for w in d['windows']]"
