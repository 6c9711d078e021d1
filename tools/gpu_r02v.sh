T=r02v
mkdir -p gpurun_out/$T
timeout 900 python -m pytest tests/test_gpu_sharded.py tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo tests rc=$?; tail -2 gpurun_out/$T/tests.log
for rep in 1 2; do for v in default prev; do
  if [ $v = default ]; then b=(); else b=(--lib build/variants/$v/libffm.so); fi
  for k in 2 5; do
    timeout 200 python bench.py "${b[@]}" --collective --workload $k --steps 20 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c${k}_${v}_$rep.json 2>/dev/null
    python -c "
import json
try:
    s=[l for l in open('gpurun_out/$T/c${k}_${v}_$rep.json') if l.startswith('{')][0]; d=json.loads(s); print('c$k $v', d['ms_per_step'], d['per_rank'][0]['ms_exchange'])
except Exception as e: print('c$k $v failed', e)"
  done
done; done
