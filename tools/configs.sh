#!/bin/bash
# All BASELINE.json configurations on one GPU (each checked against the oracle closed form),
# plus the BLS12-381 2^20 window-size sweep (config C2).  Output: one JSON line per run.
cd "$(dirname "$0")/.."
out=${1:-gpurun_out/configs.jsonl}
: > "$out"
run() { timeout 900 python bench.py --steps 3 --no-cpu-baseline "$@" 2>/dev/null | tail -1 >> "$out"; }
run --curve bn254 --log2n 10
for c in 8 10 12 13 14 15 16 17 18 20; do run --curve bls12_381 --log2n 20 --window-bits $c --no-e2e; done
run --curve bls12_381 --log2n 20
run --curve bls12_377 --log2n 24
run --curve mnt4_753 --log2n 22
run --curve bls12_381 --log2n 26
