T=r02t
mkdir -p gpurun_out/$T
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_online.py -m gpu -x -q -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo tests rc=$?; tail -2 gpurun_out/$T/tests.log
timeout 600 python bench.py --steps 10 --e2e-steps 3 --cpu-seconds 0 > gpurun_out/$T/c5.json 2> gpurun_out/$T/c5.err; echo c5 rc=$?
python -c "
import json; d=json.load(open('gpurun_out/r02t/c5.json')); print(d['ms_per_step'], d['e2e']['value'], d['e2e']['phases_s'], d['e2e']['pageable'])"
timeout 300 python bench.py --collective --steps 10 --e2e-steps 0 --cpu-seconds 0 > gpurun_out/$T/c5_coll.json 2> gpurun_out/$T/c5_coll.err; echo coll rc=$?
python -c "
import json; d=json.load(open('gpurun_out/r02t/c5_coll.json')); print(d['ms_per_step'], d['per_rank'])"
