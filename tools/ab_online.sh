for rep in 1 2; do for v in default prev; do
  if [ $v = default ]; then b=(); else b=(--lib build/variants/prev/libffm.so); fi
  timeout 300 python bench.py "${b[@]}" --workload 2 --online 4096,65536,262144 > gpurun_out/ab_online_${v}_$rep.json 2>/dev/null
  python -c "
import json
d=json.load(open('gpurun_out/ab_online_${v}_$rep.json'))
print('$v', [(w['mode'][0], w['window'], w['append_ms_median'], w['step_ms_median'], w['streamed_gbs'], w['steps_only_gbs']) for w in d['windows']])"
done; done
