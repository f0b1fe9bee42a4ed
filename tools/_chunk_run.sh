mkdir -p gpurun_out/ch
export MSM_LIB=$PWD/build_dev/libmsm_dev.so
timeout 900 python -m pytest tests/test_gpu_msm.py tests/test_gpu_multishard.py -m gpu -q -x -k "bls12_381 and (chunk or sort or heavy or headline or precompute or ragged)" > gpurun_out/ch/tests.log 2>&1; tail -5 gpurun_out/ch/tests.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/ch/bench.json 2> gpurun_out/ch/bench.err; python -c "
import json,sys; d=json.loads(open('gpurun_out/ch/bench.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], d['stages_ms'], d['e2e'], d['check']['closed_form_match'])"
