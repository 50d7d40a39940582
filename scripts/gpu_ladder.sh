python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
timeout 900 python bench.py > gpurun_out/bench_field.json 2> gpurun_out/bench_field.err; tail -2 gpurun_out/bench_field.err; cat gpurun_out/bench_field.json
run() { timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --field 0 "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
echo "full"; run
for d in 1 2 3 4; do echo "dbg $d"; OPP_PMD_DEBUG=$d run; done
echo "mh"; run --mh
