mkdir -p gpurun_out/s4
export MSM_LIB=$PWD/build_dev/libmsm_dev.so
timeout 900 python -m pytest tests/test_gpu_msm.py tests/test_gpu_multishard.py -m gpu -q -x -k "bls12_381 and (sort or heavy or headline)" > gpurun_out/s4/tests.log 2>&1; tail -5 gpurun_out/s4/tests.log
for srt in 4; do timeout 600 python bench.py --sort $srt --no-cpu-baseline --no-e2e > gpurun_out/s4/bench_sort$srt.json 2> gpurun_out/s4/bench_sort$srt.err; python -c "
import json,sys; d=json.loads(open('gpurun_out/s4/bench_sort$srt.json').read().strip().splitlines()[-1]); print($srt, d['ms_per_step'], d['stages_ms'], d['roofline_sort']['frac'], d['check'])"; done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__issue_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:k_s4 -c 3 --csv python bench.py --sort 4 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-check > gpurun_out/s4/ncu_quick.csv 2>&1; grep k_s4 gpurun_out/s4/ncu_quick.csv | cut -c1-300
