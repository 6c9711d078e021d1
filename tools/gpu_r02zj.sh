T=r02zj
mkdir -p gpurun_out/$T
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/$T/tests.log
bash tools/gpu_online2.sh $T
bash tools/gpu_ab.sh $T "2" "-" "" 1
