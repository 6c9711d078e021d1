set -x
T=r02g
mkdir -p gpurun_out/$T
timeout 1800 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/$T/gpu_tests.log 2>&1; echo tests rc=$?; tail -3 gpurun_out/$T/gpu_tests.log
bash tools/ab_variants.sh $T/ab "2 5" "golden or small_pass or digest_spec" default base default base 2>&1 | grep -v "^+"
timeout 900 compute-sanitizer --tool memcheck python tools/sanitize_smoke.py > gpurun_out/$T/san_memcheck.log 2>&1; echo memcheck rc=$?; tail -3 gpurun_out/$T/san_memcheck.log
timeout 900 compute-sanitizer --tool racecheck --num-cuda-barriers 6 python tools/sanitize_fx.py > gpurun_out/$T/san_racecheck_fx.log 2>&1; echo racecheck rc=$?; tail -12 gpurun_out/$T/san_racecheck_fx.log
timeout 600 python tools/probe_online.py 65536 8 > gpurun_out/$T/online_65536.log 2>&1; cat gpurun_out/$T/online_65536.log
