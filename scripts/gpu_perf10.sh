python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
run() { echo "== $OPP_TILE_GROUP $*"; timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
run --dh --ov 0.25; run --dh --ov 0.25 --hpass 2; run --dh --ov 0.5
OPP_TILE_GROUP=8 run; OPP_TILE_GROUP=32 run; OPP_TILE_GROUP=4 run
run --deposit 0; run --axis
