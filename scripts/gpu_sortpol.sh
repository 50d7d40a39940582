run() { timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu --field 0 "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if k in ('push_move_deposit','fill','continue','sort_move')}, d['walk']['hops_per_particle_last_step'])"; }
echo "base"; run
echo "sort10"; run --sort 10
echo "axis sort5"; run --axis
echo "axis sort10"; run --axis --sort 10
echo "axis sort20"; run --axis --sort 20
echo "hpass1"; run --hpass 1
echo "hpass0"; run --hpass 0
echo "hpass2"; run --hpass 2
