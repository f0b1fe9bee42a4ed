#!/bin/bash
# Round-end evidence at HEAD (one B200): GPU tests, smoke, default bench, configs, launch list.
cd "$(dirname "$0")/.."
o=${OUT:-gpurun_out/final2}; mkdir -p $o
timeout 900 python -m pytest tests -m gpu -x -q > $o/gpu_tests.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $o/smoke.log 2>&1
timeout 600 python bench.py > $o/bench_default.json 2> $o/bench_default.err
r() { timeout 600 python bench.py --steps 3 --check --no-cpu-baseline "$@" 2>/dev/null | tail -1 >> $o/configs.jsonl; }
r --curve bn254 --log2n 10
r --curve bls12_381 --log2n 20
r --curve bls12_381 --log2n 20 --window-bits 16 --no-e2e
r --curve bls12_377 --log2n 24
r --curve mnt4_753 --log2n 22
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 500 --csv --log-file $o/launches.csv \
  python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > $o/launches.log 2>&1
tail -3 $o/gpu_tests.log; cat $o/smoke.log | tail -2; cut -c1-300 $o/bench_default.json
