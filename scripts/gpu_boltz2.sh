# C2 step with the Boltzmann-electron Newton field solve every step
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
timeout 600 python bench.py --field-model boltzmann --no-cpu > gpurun_out/bench_boltz.json 2> gpurun_out/bench_boltz.err; tail -3 gpurun_out/bench_boltz.err; python -c "
import json; d=json.loads(open('gpurun_out/bench_boltz.json').read().strip().splitlines()[-1]); print(d['value']/1e9, d['value_incl_field']/1e9, d['field'], d['e2e'])"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_boltz.csv python bench.py --field-model boltzmann --steps 3 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu $?
