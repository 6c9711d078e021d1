#!/bin/bash
# A/B of libffm tuning variants (run under gpurun): smoke + parity subset on the default
# build, then bench.py on the given configs for each variant (build/variants/<name>).
# usage: tools/gpu_ab.sh <tag> "<configs>" [variant ...]   (variant "default" = in-tree build,
#        "env:VAR=VAL" = the in-tree build with an environment knob, "name@VAR=VAL" = both)
set -u
T=$1; CFGS=$2; shift 2
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.log 2>&1 || { echo smoke-failed; cat gpurun_out/${T}_smoke.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/${T}_parity.log 2>&1; echo "parity rc=$?"; tail -2 gpurun_out/${T}_parity.log
for v in "$@"; do
  for k in $CFGS; do
    case $v in
      default) env=();;
      env:*) env=("${v#env:}");;
      *@*) env=(FFM_LIB=build/variants/${v%@*}/libffm.so "${v#*@}");;
      *) env=(FFM_LIB=build/variants/$v/libffm.so);;
    esac
    env "${env[@]}" timeout 600 python bench.py --workload $k --steps 10 --e2e-steps 0 --cpu-seconds 0 > "gpurun_out/${T}_c${k}_${v//[:=@]/_}.json" 2> "gpurun_out/${T}_c${k}_${v//[:=@]/_}.err"
    python - "$T" "$k" "$v" <<'PY'
import json, sys
t, k, v = sys.argv[1:]
try:
    d = json.load(open(f"gpurun_out/{t}_c{k}_{v.replace(':', '_').replace('=', '_').replace('@', '_')}.json"))
    print(f"c{k} {v:10s} {d['value']:8.1f} GB/s {d['ms_per_step']:7.3f} ms  fused {d['stage_ms']['ms_fused']:.3f} ms  {d['roofline']['kernel']} frac {d['roofline']['frac']}")
except Exception as e:
    print(f"c{k} {v} failed: {e}")
PY
  done
done
echo done
