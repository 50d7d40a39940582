# particle-order policy (sort by cell vs random shuffle vs none), C2 and C5
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "shuffle" 2>&1 | tail -2
run() { timeout 600 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu --field 0 "$@" 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); p=d['phases_ms_per_step']
print('$*', round(d['value']/1e9,2), 'ms/step', round(d['ms_per_step'],3), 'pmd', round(p['push_move_deposit'],3), 'fill+sort', round(p.get('fill',0),3), 'frac', round(d['roofline']['frac'],3))"; }
run --sort 10; run --sort 0; run --sort 0 --shuffle 1; run --sort 0 --shuffle 10
run --config c5 --deposit 0 --sort 10; run --config c5 --deposit 0 --sort 0; run --config c5 --deposit 0 --sort 0 --shuffle 1
run --config c5 --deposit 1 --sort 10; run --config c5 --deposit 1 --sort 0; run --config c5 --deposit 1 --sort 0 --shuffle 1
