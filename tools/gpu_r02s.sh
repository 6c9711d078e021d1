T=r02s
mkdir -p gpurun_out/$T
timeout 300 python -m pytest tests/test_gpu_sharded.py -m gpu -x -q -p no:cacheprovider -k "nccl or two_host or eight_ranks_forced" > gpurun_out/$T/tests.log 2>&1; echo tests rc=$?; tail -2 gpurun_out/$T/tests.log
timeout 300 python -X faulthandler bench.py --collective --workload 2 --steps 10 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c2.json 2> gpurun_out/$T/c2.err; echo rc=$?; tail -30 gpurun_out/$T/c2.err; head -c 300 gpurun_out/$T/c2.json
dmesg 2>/dev/null | tail -5
