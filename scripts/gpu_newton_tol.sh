# Boltzmann solve: inner CG tolerance sweep (C2, field every step)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
for t in 1e-3 1e-4 1e-6 1e-8 1e-10 1e-11; do timeout 600 python bench.py --field-model boltzmann --newton-cg-tol $t --no-cpu --no-e2e > gpurun_out/bench_nt$t.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/bench_nt$t.json').read().strip().splitlines()[-1]); f=d['field']; print('$t', round(f['ms_per_step'],3), f['last_solve'])"; done
