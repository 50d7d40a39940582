python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
run() { echo "== $OPP_PMD_DEBUG $OPP_TILE_GROUP $*"; timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
for tg in 1 16; do export OPP_TILE_GROUP=$tg
for dbg in 1 2 3 4 0; do export OPP_PMD_DEBUG=$dbg; run --sort 5 --direct; run --sort 5; done
export OPP_PMD_DEBUG=0
run --sort 5 --direct --deposit 1; run --sort 5 --deposit 1; run --sort 0 --deposit 1; run --sort 0 --direct --deposit 1
done
export OPP_TILE_GROUP=16
timeout 900 ncu --set full --clock-control none -k regex:k_sort_move -s 2 -c 1 -o gpurun_out/prof_sortmove python bench.py --steps 12 --warmup 1 --no-e2e --no-cpu --sort 5 > /dev/null 2>&1; echo ncu $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit -s 6 -c 1 -o gpurun_out/prof_pmd_best python bench.py --steps 4 --warmup 1 --no-e2e --no-cpu --sort 5 --deposit 1 > /dev/null 2>&1; echo ncu $?
