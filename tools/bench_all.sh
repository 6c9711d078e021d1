#!/bin/bash
# All BASELINE configs at P = 1 (run under gpurun): one JSON line each into gpurun_out/<tag>_cK.json
set -u
TAG=$1
mkdir -p gpurun_out
for k in 1 2 3 4 5; do
  timeout 900 python bench.py --workload $k --steps 10 --e2e-steps 2 --cpu-seconds 10 > gpurun_out/${TAG}_c$k.json 2> gpurun_out/${TAG}_c$k.err
  timeout 600 python bench.py --workload $k --steps 10 --e2e-steps 0 --cpu-seconds 0 --two-pass > gpurun_out/${TAG}_c${k}_tp.json 2> gpurun_out/${TAG}_c${k}_tp.err
done
timeout 600 python bench.py --workload 3 --steps 5 --e2e-steps 0 --cpu-seconds 0 --digest-bits 0 > gpurun_out/${TAG}_c3_db0.json 2> gpurun_out/${TAG}_c3_db0.err
for k in 1 4 5; do
  timeout 600 python bench.py --workload $k --steps 10 --e2e-steps 0 --cpu-seconds 0 --prefilter > gpurun_out/${TAG}_c${k}_pf.json 2> gpurun_out/${TAG}_c${k}_pf.err
done
echo bench-all-done
