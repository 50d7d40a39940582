python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
run() { timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if k in ('push_move_deposit','fill')})"; }
for r in 1 2; do echo spec; run; echo nospec; OPP_PMD_DEBUG=10 run; done
