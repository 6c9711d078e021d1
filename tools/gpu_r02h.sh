set -x
T=r02h
mkdir -p gpurun_out/$T
timeout 600 compute-sanitizer --tool racecheck --racecheck-trace-sync yes --kernel-name kns=k_fused_fx python tools/san_fx_tiny.py > gpurun_out/$T/rc_trace.log 2>&1; grep -c "" gpurun_out/$T/rc_trace.log
sed -E 's/[0-9a-fx]+/N/g' gpurun_out/$T/rc_trace.log | sort | uniq -c | sort -rn | head -40
head -60 gpurun_out/$T/rc_trace.log
