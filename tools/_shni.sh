mkdir -p gpurun_out/shni
export MSM_LIB=$PWD/build_dev/libmsm_dev.so
timeout 900 python -m pytest tests/test_gpu_msm.py tests/test_gpu_multishard.py -m gpu -q -x -k "bls12_381 or bn254" > gpurun_out/shni/tests.log 2>&1; tail -3 gpurun_out/shni/tests.log
for cv in "bn254 10" "bn254 12" "bn254 14" "bls12_381 16" "bls12_381 20"; do set -- $cv
timeout 300 python bench.py --curve $1 --log2n $2 --steps 10 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > /tmp/l.json
python -c "
import json; d=json.loads(open('/tmp/l.json').read()); print('$1', $2, d['config']['window_bits'], round(d['ms_per_step'],4), d['stages_ms'].get('reduce_ms'), d['check']['closed_form_match'])"; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv python bench.py --curve bn254 --log2n 10 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-check > gpurun_out/shni/c1_launches.csv 2> /dev/null
