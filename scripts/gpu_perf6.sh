python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
run() { echo "== B$OPP_MINB P$OPP_PREFETCH $*"; timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
for mb in 1 3; do for pf in 0 1; do export OPP_MINB=$mb OPP_PREFETCH=$pf; run; done; done
export OPP_MINB=3 OPP_PREFETCH=0; run --sort 0; run --sort 2; run --axis; OPP_PMD_DEBUG=1 run; OPP_PMD_DEBUG=3 run; OPP_PMD_DEBUG=4 run
