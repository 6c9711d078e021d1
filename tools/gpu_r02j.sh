# round-2 closing check of HEAD (after the parallel append planning): smoke, the whole GPU suite, the default bench line, config 2,
# online windows, the reference arm (kernels as in r02h; the append path changed since)
T=r02j
mkdir -p gpurun_out/$T
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > gpurun_out/$T/smi.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1; echo smoke rc=$?
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/$T/gpu_tests.log 2>&1; echo tests rc=$?; tail -2 gpurun_out/$T/gpu_tests.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/$T/bench_default.json 2> gpurun_out/$T/bench_default.err; echo bench rc=$?
timeout 400 python bench.py --workload 2 --steps 20 --warmup 5 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c2.json 2> gpurun_out/$T/c2.err; echo c2 rc=$?
timeout 600 python bench.py --workload 2 --online 1,64,4096,65536,262144,524288,1000000 --check > gpurun_out/$T/c2_online.json 2> gpurun_out/$T/c2_online.err; echo online rc=$?
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/$T/reference.json 2> gpurun_out/$T/reference.err; echo ref rc=$?
python - <<'PY'
import json
for k in ("bench_default", "c2", "reference"):
    try:
        d = json.load(open(f"gpurun_out/r02j/{k}.json"))
        print(k, d.get("value"), d.get("ms_per_step"), d.get("value_device_outputs"), (d.get("roofline") or {}).get("frac"))
    except Exception as e:
        print(k, "failed", e)
d = json.load(open("gpurun_out/r02j/c2_online.json"))
for w in d["windows"]:
    print(w["mode"], w["window"], w["step_ms_median"], w["append_ms_median"], w["steps_only_gbs"], w["streamed_gbs"], w.get("parity"))
PY
