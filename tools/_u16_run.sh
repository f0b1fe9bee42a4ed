mkdir -p gpurun_out/u16
export MSM_LIB=$PWD/variants/libmsm_dev2.so
timeout 900 python -m pytest tests/test_gpu_msm.py tests/test_gpu_multishard.py -m gpu -q -x -k "(bls12_381 or bn254) and (sort or headline or chunk or split or precompute or window or ragged)" > gpurun_out/u16/tests.log 2>&1; tail -3 gpurun_out/u16/tests.log
timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/u16/bench_c4.json 2> gpurun_out/u16/bench_c4.err; python -c "
import json,sys; d=json.loads(open('gpurun_out/u16/bench_c4.json').read().strip().splitlines()[-1]); print('C4', d['ms_per_step'], d['stages_ms'], d['roofline_sort'], d['check']['closed_form_match'])"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:k_s3 -c 5 --csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-check > gpurun_out/u16/ncu_sort.csv 2>&1
