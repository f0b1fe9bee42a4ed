mkdir -p gpurun_out/c1
export MSM_LIB=$PWD/build_dev/libmsm_dev.so
timeout 900 python -m pytest tests/test_gpu_msm.py tests/test_gpu_multishard.py tests/test_gpu_layers.py -m gpu -q -x -k "bls12_381 or bn254" > gpurun_out/c1/tests.log 2>&1; tail -5 gpurun_out/c1/tests.log
timeout 300 python tools/_dbg_graph.py > gpurun_out/c1/dbg.log 2>&1; tail -3 gpurun_out/c1/dbg.log
timeout 600 python bench.py --curve bn254 --log2n 10 --steps 20 --no-cpu-baseline > gpurun_out/c1/bench_c1.json 2> gpurun_out/c1/bench_c1.err; python -c "
import json,sys; d=json.loads(open('gpurun_out/c1/bench_c1.json').read().strip().splitlines()[-1]); print('C1', d['ms_per_step'], d['stages_ms'], d['e2e']['ms_per_step'], d['check']['closed_form_match'], d['gpu_launches'])"
timeout 600 python bench.py --curve bls12_381 --log2n 20 --steps 5 --no-cpu-baseline > gpurun_out/c1/bench_c2.json 2> gpurun_out/c1/bench_c2.err; python -c "
import json,sys; d=json.loads(open('gpurun_out/c1/bench_c2.json').read().strip().splitlines()[-1]); print('C2', d['ms_per_step'], d['stages_ms'], d['check']['closed_form_match'])"
timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/c1/bench_c4.json 2> gpurun_out/c1/bench_c4.err; python -c "
import json,sys; d=json.loads(open('gpurun_out/c1/bench_c4.json').read().strip().splitlines()[-1]); print('C4', d['ms_per_step'], d['stages_ms'], d['check']['closed_form_match'])"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv python bench.py --curve bn254 --log2n 10 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-check > gpurun_out/c1/launches.csv 2> gpurun_out/c1/ncu.err
