mkdir -p gpurun_out/sm
for v in 3 4; do
  export MSM_LIB=$PWD/variants/libmsm_segminb$v.so
  timeout 900 python bench.py --curve mnt4_753 --log2n 22 --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/sm/m$v.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/sm/m$v.json').read().strip().splitlines()[-1]); print('minb $v', d['ms_per_step'], d['stages_ms']['accumulate_ms'], d['stages_ms']['reduce_ms'], d['check']['closed_form_match'])"
done
