set -x
T=r02n
mkdir -p gpurun_out/$T
timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider -k "golden or small_pass or digest_spec or flip or configs_reduced" > gpurun_out/$T/parity.log 2>&1; echo parity rc=$?; tail -3 gpurun_out/$T/parity.log
for v in default st2 st4 cw4; do
  if [ $v = default ]; then b=(); else b=(--lib build/variants/$v/libffm.so); fi
  for k in 2 5; do
    timeout 150 python bench.py "${b[@]}" --workload $k --steps 10 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c${k}_$v.json 2>/dev/null
    python -c "
import json,sys
try:
    d=json.load(open('gpurun_out/$T/c${k}_$v.json')); s=d['stage_ms']; print('c$k $v', d['ms_per_step'], 'small', s['ms_hash_small'])
except Exception as e: print('c$k $v failed', e)"
  done
done
