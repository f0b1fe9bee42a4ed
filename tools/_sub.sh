mkdir -p gpurun_out/sub
timeout 900 python -m pytest tests/test_gpu_msm.py tests/test_gpu_multishard.py -m gpu -q -x -k "pipelined or submit or chunk or graph" > gpurun_out/sub/tests.log 2>&1; tail -2 gpurun_out/sub/tests.log
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/sub/c4.json 2>gpurun_out/sub/c4.err; python -c "
import json; d=json.loads(open('gpurun_out/sub/c4.json').read().strip().splitlines()[-1]); print('C4', d['ms_per_step'], d['e2e'], d['check']['closed_form_match'])"
