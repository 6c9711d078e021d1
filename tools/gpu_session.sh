#!/bin/bash
# One GPU session (run under gpurun): quick smoke, A/B bench of the round-0 fused pass
# implementations on configs 5 and 4, then the GPU test suite.
set -u
mkdir -p gpurun_out
T=${1:-s}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${T}_smi.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.log 2>&1 || { echo smoke-failed; cat gpurun_out/${T}_smoke.log; exit 1; }
for k in 5 4; do
  for impl in 0 1; do
    FFM_FUSED_IMPL=$impl timeout 600 python bench.py --workload $k --steps 10 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/${T}_c${k}_i$impl.json 2> gpurun_out/${T}_c${k}_i$impl.err
  done
done
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/${T}_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${T}_pytest.log
tail -3 gpurun_out/${T}_pytest.log
echo done
