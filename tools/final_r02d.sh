#!/bin/bash
# Round-2 (final, d) GPU evidence, one GPU under gpurun.  Output under gpurun_out/r02d/.
cd "$(dirname "$0")/.."
o=gpurun_out/r02d; mkdir -p $o
python -m pytest tests -m gpu -q > $o/gpu_tests.log 2>&1; tail -3 $o/gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > $o/smoke.log 2>&1; tail -1 $o/smoke.log
python bench.py > $o/bench_2p26.json 2> $o/bench_2p26.err; tail -c 300 $o/bench_2p26.json
python bench.py --gpus 2 --log2n 22 --no-cpu-baseline > $o/bench_n2_shared.json 2> $o/bench_n2_shared.err
python bench.py --impl reference --steps 3 --warmup 3 > $o/bench_reference.json 2> $o/bench_reference.err
bash tools/configs.sh $o/configs.jsonl
OUT=$o/prof KERNELS="k_accumulate_sync k_bucket_segments k_finalize" bash tools/profile_round.sh
OUT=$o/prof_c1 NOLAUNCH=1 BENCH_ARGS="--curve bn254 --log2n 10" KERNELS="k_finalize" bash tools/profile_round.sh
ls -la $o
OUT=$o/prof_mnt4 NOLAUNCH=1 BENCH_ARGS="--curve mnt4_753 --log2n 22" KERNELS="k_accumulate_sync" bash tools/profile_round.sh
ls -la $o/prof_mnt4
