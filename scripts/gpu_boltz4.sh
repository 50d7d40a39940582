# Boltzmann on slabs (loopback ranks) + single-rank regression
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_multirank.py tests/test_gpu_boltzmann.py tests/test_gpu_field.py -m gpu -q -x > gpurun_out/pytest_boltz4.log 2>&1; tail -25 gpurun_out/pytest_boltz4.log
timeout 600 python bench.py --field-model boltzmann --no-cpu > gpurun_out/bench_boltz4.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/bench_boltz4.json').read().strip().splitlines()[-1]); f=d['field']; print(round(d['value']/1e9,2), round(d['value_incl_field']/1e9,2), round(f['ms_per_step'],3), f['last_solve'])"
