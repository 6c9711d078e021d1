#!/bin/bash
# quick A/B on the GPU box: targeted parity, then bench configs for env variants
# usage: tools/ab_small.sh <tag> "<configs>" "<pytest -k expr>" [ENV=VAL ...]   ("-" = default env)
set -u
T=$1; CFGS=$2; KX=$3; shift 3
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.log 2>&1 || { echo smoke-failed; tail -20 gpurun_out/${T}_smoke.log; exit 1; }
if [ "$KX" != "-" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q -k "$KX" > gpurun_out/${T}_parity.log 2>&1; echo "parity rc=$?"; tail -3 gpurun_out/${T}_parity.log
fi
n=0
for v in "$@"; do
  n=$((n+1))
  for k in $CFGS; do
    if [ "$v" = "-" ]; then e=(); else e=($v); fi
    out="gpurun_out/${T}_c${k}_v${n}.json"
    env "${e[@]}" timeout 600 python bench.py --workload $k --steps 10 --e2e-steps 0 --cpu-seconds 0 > "$out" 2> "${out%.json}.err"
    python - "$out" "$k" "$v" <<'PY'
import json, sys
out, k, v = sys.argv[1:]
try:
    d = json.load(open(out))
    s = d['stage_ms']
    print(f"c{k} {v[-34:]:34s} {d['value']:8.1f} GB/s {d['ms_per_step']:7.3f} ms | small {s['ms_hash_small']:.3f} group {s['ms_group']:.3f} fused {s['ms_fused']:.3f} label {s['ms_label']:.3f} | {d['roofline']['kernel']} frac {d['roofline']['frac']}")
except Exception as e:
    print(f"c{k} {v} failed: {e}"); print(open(out.replace('.json', '.err')).read()[-1500:])
PY
  done
done
echo done
