#!/bin/bash
# Build BLS12-381-only variant libraries for A/B timing (other curves reuse build/ objects).
set -e
cd "$(dirname "$0")/.."
mkdir -p variants
build_variant() {  # name, defines...
  name=$1; shift
  args=()
  for d in "$@"; do args+=(-D "$d"); done
  python tools/build.py --dev bls12_381 --build-dir build/v_$name --out variants/libmsm_$name.so "${args[@]}" > /tmp/bv_$name.log 2>&1 || { echo "FAIL $name"; tail -5 /tmp/bv_$name.log; }
  grep -A3 "k_accumulate" build/v_$name/curve_bls12_381.o.log | grep -E "Used|spill" | tr '\n' ' '; echo " <- $name"
}
for spec in "$@"; do
  IFS=':' read -r -a parts <<< "$spec"
  build_variant "${parts[@]}" &
done
wait
