python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
run() { echo "== R$OPP_REFILL B$OPP_MINB $*"; timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
export OPP_TILE_GROUP=16
for rf in 0 1; do for mb in 1 3; do export OPP_REFILL=$rf OPP_MINB=$mb
run --sort 5 --deposit 1; run --sort 5 --deposit 1 --dh --ov 0.25
done; done
export OPP_REFILL=0 OPP_MINB=1
run --sort 0 --deposit 1
