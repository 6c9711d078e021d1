#!/bin/bash
# A/B of the working tree against build/variants/<v>/libffm.so builds on the GPU box.
# usage: tools/gpu_ab.sh <tag> "<configs>" "<pytest -k expr or ->" "<variants>" [reps]
set -u
T=$1; CFGS=$2; KX=$3; VARS=$4; REPS=${5:-2}
mkdir -p gpurun_out/$T
if [ "$KX" != "-" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider -k "$KX" > gpurun_out/$T/tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/$T/tests.log
fi
for rep in $(seq 1 $REPS); do for v in default $VARS; do
  if [ $v = default ]; then b=(); else b=(--lib build/variants/$v/libffm.so); fi
  for k in $CFGS; do
    out=gpurun_out/$T/c${k}_${v}_$rep.json
    timeout 300 python bench.py "${b[@]}" --workload $k --steps 20 --e2e-steps 0 --cpu-seconds 0 > $out 2>${out%.json}.err
    python - "$out" "$k" "$v" <<'PY'
import json, sys
out, k, v = sys.argv[1:]
try:
    d = json.load(open(out)); s = d['stage_ms']
    print(f"c{k} {v:12s} {d['ms_per_step']:8.4f} ms (dev out {d['ms_per_step_device_outputs']:8.4f}) small {s['ms_hash_small']:.4f} group {s['ms_group']:.4f} fused {s['ms_fused']:.4f} label {s['ms_label']:.4f}")
except Exception as e:
    print(f"c{k} {v} failed: {e}"); print(open(out.replace('.json', '.err')).read()[-1500:])
PY
  done
done; done
