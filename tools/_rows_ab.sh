mkdir -p gpurun_out/rows
export MSM_LIB=$PWD/variants/libmsm_rows.so
timeout 600 python -m pytest tests/test_gpu_layers.py tests/test_gpu_msm.py -m gpu -q -x -k "mnt4" > gpurun_out/rows/tests.log 2>&1; tail -3 gpurun_out/rows/tests.log
for v in rows main; do
  if [ $v = main ]; then unset MSM_LIB; fi
  timeout 900 python bench.py --curve mnt4_753 --log2n 22 --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/rows/$v.json 2> gpurun_out/rows/$v.err
  python -c "
import json; d=json.loads(open('gpurun_out/rows/$v.json').read().strip().splitlines()[-1]); print('$v', d['ms_per_step'], d['stages_ms'], d['roofline']['frac'], d['check']['closed_form_match'])"
done
export MSM_LIB=$PWD/variants/libmsm_segsync.so
timeout 900 python bench.py --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/rows/segsync.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/rows/segsync.json').read().strip().splitlines()[-1]); print('segsync C4', d['ms_per_step'], d['stages_ms']['reduce_ms'], d['check']['closed_form_match'])"
