#!/bin/bash
# Parity subset + bench per libffm variant (build/variants/<name>; "default" = in-tree).
# usage: tools/ab_variants.sh <tag> "<configs>" "<pytest -k expr>" variant ...
set -u
T=$1; CFGS=$2; KX=$3; shift 3
mkdir -p gpurun_out
for v in "$@"; do
  if [ "$v" = default ]; then e=(); else e=(--ffm-lib build/variants/$v/libffm.so); fi
  timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "$KX" "${e[@]}" > gpurun_out/${T}_${v}_parity.log 2>&1
  echo "$v parity rc=$? $(tail -1 gpurun_out/${T}_${v}_parity.log)"
  for k in $CFGS; do
    out=gpurun_out/${T}_c${k}_${v}.json
    if [ "$v" = default ]; then b=(); else b=(--lib build/variants/$v/libffm.so); fi
    timeout 600 python bench.py "${b[@]}" --workload $k --steps 10 --e2e-steps 0 --cpu-seconds 0 > $out 2> ${out%.json}.err
    python - "$out" "$k" "$v" <<'PY'
import json, sys
out, k, v = sys.argv[1:]
try:
    d = json.load(open(out)); s = d['stage_ms']
    print(f"c{k} {v:14s} {d['value']:8.1f} GB/s {d['ms_per_step']:7.3f} ms | small {s['ms_hash_small']:.3f} group {s['ms_group']:.3f} fused {s['ms_fused']:.3f}")
except Exception as e:
    print(f"c{k} {v} failed: {e}"); print(open(out.replace('.json', '.err')).read()[-1500:])
PY
  done
done
