# round 2 check: GPU tests, config 2 / 5 bench lines, online-mode measurement
set -x
T=r02c
mkdir -p gpurun_out/$T
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1; echo smoke rc=$?
timeout 1800 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/$T/gpu_tests.log 2>&1; echo tests rc=$?
tail -30 gpurun_out/$T/gpu_tests.log
timeout 600 python bench.py --workload 2 --steps 20 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c2.json 2> gpurun_out/$T/c2.err; echo c2 rc=$?
timeout 900 python bench.py --workload 2 --online 1,64,4096,65536 --check > gpurun_out/$T/c2_online.json 2> gpurun_out/$T/c2_online.err; echo online rc=$?
tail -c 2500 gpurun_out/$T/c2_online.json
timeout 900 python bench.py --steps 20 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c5.json 2> gpurun_out/$T/c5.err; echo c5 rc=$?
python - <<'PY'
import json
for k in ("c2", "c5"):
    try:
        d = json.load(open(f"gpurun_out/r02c/{k}.json"))
        print(k, d["ms_per_step"], d["ms_per_step_device_outputs"], d["value"], d["stage_ms"])
    except Exception as e:
        print(k, "failed", e)
PY
