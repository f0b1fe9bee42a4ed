set -x
mkdir -p gpurun_out
export MSM_LIB=$PWD/variants/libmsm_bgcd.so
timeout 600 python -m pytest tests/test_gpu_layers.py -q -m gpu -k "bls12_381" -x 2>&1 | tail -5 > gpurun_out/bgcd_tests.log
for n in 20 26; do timeout 300 python bench.py --log2n $n --steps 5 --warmup 3 --no-cpu-baseline --check >> gpurun_out/bgcd_bench.jsonl 2>gpurun_out/bgcd_bench_$n.err; done
unset MSM_LIB
timeout 300 python bench.py --log2n 20 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --check >> gpurun_out/base_bench.jsonl 2>gpurun_out/base_bench.err
cat gpurun_out/bgcd_tests.log
