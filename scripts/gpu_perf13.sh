python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "dh or every_particle" 2>&1 | tail -3
run() { echo "== $*"; timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()}, d['walk'])"; }
run; run --sort 10; run --sort 3
