T=r02z9
mkdir -p gpurun_out/$T
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider -k "golden or small or configs_reduced or flip or random or online or prefilter or channel" > gpurun_out/$T/tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/$T/tests.log
bash tools/gpu_ab.sh $T "2 5 1" "-" "prev" 2
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/$T/c2_launches.csv python bench.py --workload 2 --steps 2 --warmup 3 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c2_ncu.log 2>&1
python tools/ncu_launch_table.py gpurun_out/$T/c2_launches.csv | head -12
