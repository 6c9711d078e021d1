set -x
T=r02i
mkdir -p gpurun_out/$T
timeout 600 compute-sanitizer --tool racecheck python tools/san_fx_tiny.py > gpurun_out/$T/rc_tiny.log 2>&1; tail -4 gpurun_out/$T/rc_tiny.log
timeout 900 compute-sanitizer --tool racecheck python tools/sanitize_fx.py > gpurun_out/$T/rc_fx.log 2>&1; tail -6 gpurun_out/$T/rc_fx.log
bash tools/ab_variants.sh $T/ab "5 4" "golden or flip or difference or two_pass or configs_reduced" default arrive1 default arrive1 2>&1 | grep -v "^+"
