# C3 e2e with overlapped copies
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
timeout 600 python bench.py --config c3 --no-cpu > gpurun_out/bench_c3e2e.json 2> gpurun_out/bench_c3e2e.err; tail -2 gpurun_out/bench_c3e2e.err; python -c "
import json; d=json.loads(open('gpurun_out/bench_c3e2e.json').read().strip().splitlines()[-1]); print(round(d['value']/1e9,3), d['e2e'])"
