# A/B of the role-split small pass (k_small_role) against the mixed octet kernel and tuning variants
set -x
T=r02e
mkdir -p gpurun_out/$T
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider > gpurun_out/$T/parity_default.log 2>&1; echo parity rc=$?; tail -3 gpurun_out/$T/parity_default.log
bash tools/ab_variants.sh $T/ab "2 5" "golden or random_tiny or small_pass or digest_spec or flip or configs_reduced" default nosplit cj4 hj2 s3 t256 2>&1 | grep -v "^+"
