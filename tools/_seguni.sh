mkdir -p gpurun_out/seguni
MSM_LIB=$PWD/variants/libmsm_seguni.so timeout 900 python bench.py --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/seguni/c4.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/seguni/c4.json').read().strip().splitlines()[-1]); print('seguni C4', d['ms_per_step'], d['stages_ms'], d['check']['closed_form_match'])"
MSM_LIB=$PWD/variants/libmsm_seguni.so timeout 900 python bench.py --log2n 20 --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/seguni/c2.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/seguni/c2.json').read().strip().splitlines()[-1]); print('seguni C2', d['ms_per_step'], d['stages_ms'], d['check']['closed_form_match'])"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv python bench.py --curve bn254 --log2n 10 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-check > gpurun_out/seguni/c1_launches.csv 2> /dev/null
