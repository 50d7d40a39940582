python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
run() { echo "== $*"; timeout 300 python bench.py --steps 30 --warmup 3 --no-e2e --no-cpu "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if k in ('push_move_deposit','fill','sort_count','sort_move')})"; }
echo base; run
for pg in "3 4" "3 8" "2 4" "4 4" "3 3" "2 8"; do set -- $pg; echo "passes $1 grid $2"; OPP_SORT_PASSES=$1 OPP_SORT_GRID=$2 run; done
echo base; run
