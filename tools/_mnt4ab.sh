mkdir -p gpurun_out/mab
for v in main lat; do
  if [ $v = lat ]; then export MSM_LIB=$PWD/variants/libmsm_mnt4lat.so; else unset MSM_LIB; fi
  timeout 900 python bench.py --curve mnt4_753 --log2n 22 --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/mab/$v.json 2> gpurun_out/mab/$v.err
  python -c "
import json; d=json.loads(open('gpurun_out/mab/$v.json').read().strip().splitlines()[-1]); print('$v', d['ms_per_step'], d['stages_ms']['accumulate_ms'], d['stages_ms']['reduce_ms'], d['check']['closed_form_match'])"
done
unset MSM_LIB
for c in 6 8 10 12 14; do timeout 300 python bench.py --curve bn254 --log2n 10 --window-bits $c --steps 20 --no-cpu-baseline --no-e2e > gpurun_out/mab/c1_$c.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/mab/c1_$c.json').read().strip().splitlines()[-1]); print('C1 c=$c', d['ms_per_step'], d['check']['closed_form_match'])"; done
MSM_NO_GRAPH=1 timeout 300 python bench.py --curve bn254 --log2n 10 --steps 20 --no-cpu-baseline --no-e2e > gpurun_out/mab/c1_nograph.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/mab/c1_nograph.json').read().strip().splitlines()[-1]); print('C1 nograph', d['ms_per_step'], d['stages_ms'])"
