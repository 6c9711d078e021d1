set -x
mkdir -p gpurun_out/r02a
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r02a/smi.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02a/smoke.log 2>&1; echo smoke rc=$?
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/r02a/gpu_tests.log 2>&1; echo tests rc=$?
tail -30 gpurun_out/r02a/gpu_tests.log
timeout 600 python bench.py --gpus 4 --same-device --workload 5 --n-scale 0.1 --check --steps 5 --e2e-steps 2 --e2e-pageable 0 --cpu-seconds 0 > gpurun_out/r02a/bench_4same.json 2> gpurun_out/r02a/bench_4same.err; echo b4 rc=$?
tail -c 1500 gpurun_out/r02a/bench_4same.json; tail -5 gpurun_out/r02a/bench_4same.err
timeout 900 python bench.py --steps 10 > gpurun_out/r02a/bench_default.json 2> gpurun_out/r02a/bench_default.err; echo b1 rc=$?
tail -c 3000 gpurun_out/r02a/bench_default.json; tail -5 gpurun_out/r02a/bench_default.err
