# Boltzmann: cold-start stopping reference (reading B4), warm starts 1 / 2
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_boltzmann.py -m gpu -q -s -x > gpurun_out/pytest_boltz3.log 2>&1; tail -4 gpurun_out/pytest_boltz3.log
for w in 1 2; do timeout 600 python bench.py --field-model boltzmann --cg-warm $w --no-cpu > gpurun_out/bench_boltz3_w$w.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/bench_boltz3_w$w.json').read().strip().splitlines()[-1]); f=d['field']; print($w, round(d['value']/1e9,2), round(d['value_incl_field']/1e9,2), round(f['ms_per_step'],3), f['last_solve'])"; done
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
