# C3: sort by cell every K steps (sort inside the timed step) vs never
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
for k in 0 4 8 16 32; do timeout 600 python bench.py --config c3 --em-sort $k --no-cpu --no-e2e --steps 32 > gpurun_out/bench_emsort$k.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/bench_emsort$k.json').read().strip().splitlines()[-1]); print($k, round(d['value']/1e9,3), d['ms_per_step'], d['roofline']['frac'])"; done
