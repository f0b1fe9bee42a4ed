mkdir -p gpurun_out/sw
: > gpurun_out/sw/sweep.txt
for cv in "bn254 10" "bn254 12" "bn254 14" "bn254 16" "bls12_381 16" "bls12_381 18"; do
  set -- $cv
  for c in 4 5 6 7 8 10 12 14 16; do
    timeout 300 python bench.py --curve $1 --log2n $2 --window-bits $c --steps 10 --no-cpu-baseline --no-e2e --no-check 2>/dev/null | tail -1 > /tmp/l.json
    python -c "
import json; d=json.loads(open('/tmp/l.json').read()); print('$1', $2, $c, round(d['ms_per_step'],4))" >> gpurun_out/sw/sweep.txt
  done
  timeout 300 python bench.py --curve $1 --log2n $2 --steps 10 --no-cpu-baseline --no-e2e --no-check 2>/dev/null | tail -1 > /tmp/l.json
  python -c "
import json; d=json.loads(open('/tmp/l.json').read()); print('$1', $2, 'auto', d['config']['window_bits'], round(d['ms_per_step'],4))" >> gpurun_out/sw/sweep.txt
done
cat gpurun_out/sw/sweep.txt
