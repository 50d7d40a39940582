python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
run() { echo "== $*"; timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if k in ('push_move_deposit','fill','sort_count','sort_move')})"; }
run
for p in 2 3 7; do echo "passes $p"; OPP_SORT_PASSES=$p run; done
for g in 2 4 16; do echo "grid $g"; OPP_SORT_GRID=$g run; done
echo "passes 3 grid 4"; OPP_SORT_PASSES=3 OPP_SORT_GRID=4 run
