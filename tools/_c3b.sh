for c in 22 23; do timeout 600 python bench.py --curve bls12_377 --log2n 24 --window-bits $c --steps 5 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > /tmp/l.json; python -c "
import json; d=json.loads(open('/tmp/l.json').read()); print('C3 c=$c', round(d['ms_per_step'],2), d['stages_ms']['accumulate_ms'], d['stages_ms']['reduce_ms'], d['stages_ms']['sort_ms'], d['check']['closed_form_match'])"; done
for c in 21 22 23 24; do timeout 600 python bench.py --curve bls12_377 --log2n 22 --window-bits $c --steps 5 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > /tmp/l.json; python -c "
import json; d=json.loads(open('/tmp/l.json').read()); print('377 2^22 c=$c', round(d['ms_per_step'],2), d['check']['closed_form_match'])"; done
