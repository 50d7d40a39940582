python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 900 python scripts/debug_mr4.py 2>&1 | tail -4
run() { echo "== $*"; timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
export OPP_TILE_GROUP=16
run --sort 5 --deposit 1; run --sort 5 --deposit 1 --direct; run --sort 0 --deposit 1; run --sort 2 --deposit 1
OPP_PMD_DEBUG=1 run --sort 5 --deposit 1; OPP_PMD_DEBUG=3 run --sort 5 --deposit 1; OPP_PMD_DEBUG=4 run --sort 5 --deposit 1
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
