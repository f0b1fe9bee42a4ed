mkdir -p gpurun_out/dig
export MSM_LIB=$PWD/variants/libmsm_dig.so
timeout 900 python -m pytest tests/test_gpu_msm.py tests/test_gpu_multishard.py tests/test_gpu_layers.py -m gpu -q -x -k "(bls12_381 or bn254) and (sort or digit or heavy or headline or split or chunk or window)" > gpurun_out/dig/tests.log 2>&1; tail -2 gpurun_out/dig/tests.log
timeout 600 python bench.py --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/dig/c4.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/dig/c4.json').read().strip().splitlines()[-1]); print('dig C4', d['ms_per_step'], d['stages_ms'], d['check']['closed_form_match'])"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_s3_ -c 5 --csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-check > gpurun_out/dig/ncu_sort.csv 2>/dev/null
