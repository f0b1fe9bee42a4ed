#!/bin/bash
# A/B + full GPU tests of the warp-tree k_sum_groups build (variants/libmsm_sw.so)
cd "$(dirname "$0")/.."
o=gpurun_out/sw; mkdir -p $o
L=${SWLIB:-variants/libmsm_sw.so}
export MSM_LIB=$PWD/$L
r() { timeout 600 python bench.py --steps 5 --check --no-cpu-baseline --no-e2e "$@" 2>/dev/null | tail -1 >> $o/bench_sw.jsonl; }
r --log2n 20; r --log2n 26
[ -n "$FULL" ] && { r --curve bn254 --log2n 10; r --curve bls12_377 --log2n 24; r --curve mnt4_753 --log2n 22; }
[ -n "$FULL" ] && timeout 900 python -m pytest tests -m gpu -x -q > $o/gpu_tests.log 2>&1
[ -n "$FULL" ] && timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $o/smoke.log 2>&1
unset MSM_LIB
[ -n "$FULL" ] && timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 500 --csv --log-file $o/launches.csv \
  env MSM_LIB=$PWD/$L python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > $o/launches.log 2>&1
tail -3 $o/gpu_tests.log 2>/dev/null; cut -c1-200 $o/bench_sw.jsonl
