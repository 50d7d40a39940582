python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
run() { timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu --field 0 "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if k in ('push_move_deposit','fill','continue','sort_move')}, d['walk']['hops_per_particle_last_step'])"; }
echo "ov16 sort10"; run
echo "ov32 sort10"; OPP_OV_COMPACT=0 run
echo "ov16 sort8"; run --sort 8
echo "ov16 sort12"; run --sort 12
echo "ov16 sort15"; run --sort 15
echo "ov16 h/16"; run --ov 0.0625
echo "ov16 h/4"; run --ov 0.25
