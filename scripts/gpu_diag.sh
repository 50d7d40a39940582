python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 600 python -m pytest tests/test_gpu_multirank.py -x -q 2>&1 | grep -vE "^\s*$" | tail -30
run() { echo "== $*"; timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
export OPP_TILE_GROUP=1
for dbg in 1 2 3 4 0; do export OPP_PMD_DEBUG=$dbg; run --sort 0 --direct; run --sort 5 --direct; done
