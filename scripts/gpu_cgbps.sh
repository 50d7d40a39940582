# field CG: blocks per SM (1: R = 5 rows per thread, 2: R = 3)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_field.py -m gpu -q -x > gpurun_out/pytest_cgbps.log 2>&1; tail -2 gpurun_out/pytest_cgbps.log
for b in 2; do OPP_CG_BPS=$b timeout 600 python bench.py --no-cpu --no-e2e > gpurun_out/bench_cgbps$b.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/bench_cgbps$b.json').read().strip().splitlines()[-1]); f=d['field']; print('bps=$b', round(d['value_incl_field']/1e9,2), round(f['ms_per_step'],3), f['cg_iterations_last'])"; done
OPP_CG_BPS=1 timeout 900 python -m pytest tests/test_gpu_field.py tests/test_gpu_boltzmann.py -m gpu -q -x > gpurun_out/pytest_cgbps1.log 2>&1; tail -2 gpurun_out/pytest_cgbps1.log
