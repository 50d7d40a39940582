# field CG: row vectors in shared memory (k_pcg_reg, OPP_CG_REG=1) vs k_pcg
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_field.py tests/test_gpu_boltzmann.py -m gpu -q -x > gpurun_out/pytest_cgreg.log 2>&1; tail -3 gpurun_out/pytest_cgreg.log
for r in 0 1; do OPP_CG_REG=$r timeout 600 python bench.py --no-cpu --no-e2e > gpurun_out/bench_cgreg$r.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/bench_cgreg$r.json').read().strip().splitlines()[-1]); f=d['field']; print('reg=$r', round(d['value']/1e9,2), round(d['value_incl_field']/1e9,2), round(f['ms_per_step'],3), f['cg_iterations_last'])"; done
OPP_CG_REG=1 timeout 600 python bench.py --field-model boltzmann --no-cpu --no-e2e > gpurun_out/bench_cgreg_bz.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/bench_cgreg_bz.json').read().strip().splitlines()[-1]); f=d['field']; print('bz reg=1', round(d['value_incl_field']/1e9,2), round(f['ms_per_step'],3), f['last_solve'])"
