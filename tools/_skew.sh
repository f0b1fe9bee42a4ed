mkdir -p gpurun_out/skew
for v in 6 13; do
  export MSM_LIB=$PWD/variants/libmsm_skew$v.so
  timeout 600 python -m pytest tests/test_gpu_layers.py tests/test_gpu_msm.py -m gpu -q -x -k "bls12_381 and (field or ec or ragged or precompute)" > gpurun_out/skew/t$v.log 2>&1; tail -1 gpurun_out/skew/t$v.log
  timeout 600 python bench.py --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/skew/c4_$v.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/skew/c4_$v.json').read().strip().splitlines()[-1]); print('skew $v C4', d['ms_per_step'], d['stages_ms']['accumulate_ms'], d['roofline']['frac'], d['check']['closed_form_match'])"
done
