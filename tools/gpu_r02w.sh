T=r02x
mkdir -p gpurun_out/$T
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "golden or small or configs_reduced or flip or random" -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo tests rc=$?; tail -2 gpurun_out/$T/tests.log
for rep in 1 2; do for v in default prev; do
  if [ $v = default ]; then b=(); else b=(--lib build/variants/$v/libffm.so); fi
  for k in 2 5; do
    timeout 200 python bench.py "${b[@]}" --workload $k --steps 20 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c${k}_${v}_$rep.json 2>/dev/null
    python -c "
import json
try:
    d=json.load(open('gpurun_out/$T/c${k}_${v}_$rep.json')); s=d['stage_ms']; print('c$k $v', d['ms_per_step'], d['ms_per_step_device_outputs'], 'small', s['ms_hash_small'])
except Exception as e: print('c$k $v failed', e)"
  done
done; done
