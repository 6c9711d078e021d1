T=r02y
mkdir -p gpurun_out/$T
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1; echo smoke rc=$?; tail -1 gpurun_out/$T/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo tests rc=$?; tail -2 gpurun_out/$T/tests.log
timeout 300 python bench.py > gpurun_out/$T/default.json 2> gpurun_out/$T/default.err; echo default rc=$?; head -c 600 gpurun_out/$T/default.json
for k in 2 1 3 4; do
  timeout 200 python bench.py --workload $k --steps 20 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c$k.json 2>/dev/null
  python -c "
import json
d=json.load(open('gpurun_out/$T/c$k.json')); s=d['stage_ms']; print('c$k', d['ms_per_step'], d['ms_per_step_device_outputs'], s)"
done
