T=r02zi
mkdir -p gpurun_out/$T
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider -k "golden or small or configs_reduced or flip or random or online" > gpurun_out/$T/tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/$T/tests.log
bash tools/gpu_ab.sh $T "2 5" "-" "prev" 2
bash tools/gpu_online2.sh $T
