# linear CG: extrapolated warm start (warm_start 2) vs last solution
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_field.py -m gpu -q -x -k "extrapolated or matches" > gpurun_out/pytest_warm2.log 2>&1; tail -3 gpurun_out/pytest_warm2.log
for w in 1 2; do timeout 600 python bench.py --cg-warm $w --no-cpu --no-e2e > gpurun_out/bench_warm$w.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/bench_warm$w.json').read().strip().splitlines()[-1]); print($w, d['value']/1e9, d['value_incl_field']/1e9, d['field']['ms_per_step'], d['field']['cg_iterations_last'])"; done
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
