# round-2 final check (HEAD): GPU suite, bench lines of every config, online, same-GPU 8 ranks,
# ncu launch lists + full-set captures, sanitizers, reference arm
set -x
T=r02h
mkdir -p gpurun_out/$T
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > gpurun_out/$T/smi.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1; echo smoke rc=$?
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/$T/gpu_tests.log 2>&1; echo tests rc=$?; tail -3 gpurun_out/$T/gpu_tests.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/$T/bench_default.json 2> gpurun_out/$T/bench_default.err; echo bench rc=$?
for k in 1 2 3 4; do timeout 400 python bench.py --workload $k --steps 20 --warmup 5 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c$k.json 2> gpurun_out/$T/c$k.err; echo c$k rc=$?; done
timeout 600 python bench.py --workload 2 --online 1,64,4096,65536,262144,524288,1000000 --check > gpurun_out/$T/c2_online.json 2> gpurun_out/$T/c2_online.err; echo online rc=$?
timeout 900 python bench.py --gpus 8 --same-device --workload 5 --n-scale 0.05 --check --steps 5 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/same8.json 2> gpurun_out/$T/same8.err; echo same8 rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/$T/c5_launches.csv python bench.py --steps 2 --warmup 3 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c5_launch.log 2>&1; echo l5 rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/$T/c2_launches.csv python bench.py --workload 2 --steps 2 --warmup 3 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c2_launch.log 2>&1; echo l2 rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_fused_fx|k_fused_small|k_prefix_hash|k_group_insert|k_leader0|k_label_hist|k_fx_fill|k_hash_combine|k_spec_label" -s 12 -c 12 -o gpurun_out/$T/c5_prof python bench.py --steps 1 --warmup 3 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c5_prof.log 2>&1; echo p5 rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_fused_small|k_group_insert|k_leader0|k_label_hist|k_leader0_label|k_spec_label" -s 8 -c 5 -o gpurun_out/$T/c2_prof python bench.py --workload 2 --steps 1 --warmup 3 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c2_prof.log 2>&1; echo p2 rc=$?
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/$T/reference.json 2> gpurun_out/$T/reference.err; echo ref rc=$?
python - <<'PY'
import json
for k in ("bench_default", "c1", "c2", "c3", "c4", "same8", "reference"):
    try:
        d = json.load(open(f"gpurun_out/r02h/{k}.json"))
        print(k, d.get("value"), d.get("ms_per_step"), d.get("value_device_outputs"), (d.get("roofline") or {}).get("frac"), d.get("parity"))
    except Exception as e:
        print(k, "failed", e)
PY
