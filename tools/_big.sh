mkdir -p gpurun_out/big
export MSM_LIB=$PWD/build_dev/libmsm_dev.so
timeout 900 python -m pytest tests/test_gpu_msm.py tests/test_gpu_multishard.py -m gpu -q -x -k "(bls12_381 or bn254) and (sort or heavy or headline or chunk or skew or precompute)" > gpurun_out/big/tests.log 2>&1; tail -2 gpurun_out/big/tests.log
for c in 14 15 16 17 18; do timeout 600 python bench.py --log2n 20 --window-bits $c --steps 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > /tmp/l.json; python -c "
import json; d=json.loads(open('/tmp/l.json').read()); print('C2 c=$c', round(d['ms_per_step'],3), d['stages_ms']['accumulate_ms'], d['stages_ms']['reduce_ms'], d['stages_ms']['sort_ms'], d['check']['closed_form_match'])"; done
for c in 22 23; do timeout 600 python bench.py --log2n 24 --window-bits $c --steps 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > /tmp/l.json; python -c "
import json; d=json.loads(open('/tmp/l.json').read()); print('2^24 c=$c', round(d['ms_per_step'],2), d['stages_ms']['accumulate_ms'], d['stages_ms']['reduce_ms'], d['stages_ms']['sort_ms'], d['check']['closed_form_match'])"; done
timeout 600 python bench.py --steps 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > /tmp/l.json; python -c "
import json; d=json.loads(open('/tmp/l.json').read()); print('C4', round(d['ms_per_step'],2), d['stages_ms']['sort_ms'], d['check']['closed_form_match'])"
unset MSM_LIB
for n in pf2 sync pf0; do MSM_LIB=$PWD/variants/libmsm_m$n.so timeout 900 python bench.py --curve mnt4_753 --log2n 22 --steps 2 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > /tmp/l.json; python -c "
import json; d=json.loads(open('/tmp/l.json').read()); print('mnt4 $n', round(d['ms_per_step'],2), d['stages_ms']['accumulate_ms'], d['stages_ms']['reduce_ms'], d['check']['closed_form_match'])"; done
